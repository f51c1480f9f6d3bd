#!/usr/bin/env bash
# Capture the round's profiling evidence on the GPU box (run under gpurun, 1 GPU):
#   1. launch list (cold, serialised) of one cfg3 bench step  -> gpurun_out/launches_<tag>_<cfg>.csv
#   2. ncu --set full of the top kernels at cfg3               -> gpurun_out/prof_<tag>_<cfg>_<k>.ncu-rep
# Numbers printed under ncu are never bench values.
#   scripts/profile_round.sh TAG [CFG] [kernels...]
set -u
TAG=${1:-r01}
CFG=${2:-cfg3}
shift 2 2>/dev/null
KS=${@:-scatter_table refine bucket_join greedy_accept}
mkdir -p gpurun_out
export BENCH_ALLOW_SHORT_WARMUP=1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
if [ -z "${NO_LAUNCHES:-}" ]; then
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv \
    --log-file gpurun_out/launches_${TAG}_${CFG}.csv \
    python bench.py --config $CFG --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/launches_${TAG}.log 2>&1
fi
for k in $KS; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s 1 -c 1 \
      -o gpurun_out/prof_${TAG}_${CFG}_${k} \
      python bench.py --config $CFG --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_${TAG}_${k}.log 2>&1
done
ls -la gpurun_out
