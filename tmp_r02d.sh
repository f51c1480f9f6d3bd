PYTEST_TIMEOUT=1500 NO_BENCH=1 bash scripts/gpu_check.sh r02d "gpu and not slow"
bash scripts/gpu_ab_env.sh r02j 2 "warp=X=0" "bulk=LASAGNA_JOIN=bulk"
BENCH_ARGS="--lengths-per-pass 19" bash scripts/gpu_ab_env.sh r02p 1 "lpp19=X=0"
BENCH_ARGS="--lengths-per-pass 13" bash scripts/gpu_ab_env.sh r02p 1 "lpp13=X=0"
