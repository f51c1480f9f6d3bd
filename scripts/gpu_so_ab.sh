#!/usr/bin/env bash
# A/B of prebuilt liblasagna.so variants (scratch/lib_<name>.so) on one box, interleaved:
#   scripts/gpu_so_ab.sh TAG name1 name2 ...     (each bench run: --no-cpu-baseline)
set -u
TAG=$1; shift
mkdir -p gpurun_out
SO=paper_conf_ipps_goswamilsp18_b200/liblasagna.so
for rep in 1 2; do
  for v in "$@"; do
    cp scratch/lib_$v.so $SO
    timeout 600 python bench.py --no-cpu-baseline ${BENCH_ARGS:-} > gpurun_out/bench_${TAG}_${v}_$rep.log 2>&1
    echo "$v/$rep: $(tail -1 gpurun_out/bench_${TAG}_${v}_$rep.log | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["ms_per_step"],2), {k: round(v["ms_per_step"],2) for k,v in d["roofline"]["phases"].items()}, round(d["e2e"]["ms_per_step"],1))' 2>&1)" >> gpurun_out/status_${TAG}.txt
  done
done
cat gpurun_out/status_${TAG}.txt
