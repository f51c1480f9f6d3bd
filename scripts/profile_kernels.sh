#!/usr/bin/env bash
# ncu --set full of selected kernels (regexes) at a config: scripts/profile_kernels.sh TAG CFG k1 k2 ...
set -u
TAG=$1; CFG=$2; shift 2
mkdir -p gpurun_out
export BENCH_ALLOW_SHORT_WARMUP=1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for k in "$@"; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s 1 -c 1 \
      -o gpurun_out/prof_${TAG}_${CFG}_${k} \
      python bench.py --config $CFG --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_${TAG}_${k}.log 2>&1
done
ls gpurun_out | grep prof_${TAG}
