bash scripts/gpu_ab_env.sh r02f 1 "warp=X=0" "bulk=LASAGNA_JOIN=bulk"
BENCH_ARGS="--lengths-per-pass 19" bash scripts/gpu_ab_env.sh r02f 1 "lpp19=X=0"
BENCH_ARGS="--lengths-per-pass 13" bash scripts/gpu_ab_env.sh r02f 1 "lpp13=X=0"
