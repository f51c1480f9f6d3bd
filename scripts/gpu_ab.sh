#!/usr/bin/env bash
# A/B on the GPU box: build, a pytest selection, then bench.py once per env setting.
#   scripts/gpu_ab.sh TAG "pytest -k expr" "ENV1=a" "ENV1=b" ...
set -u
TAG=$1; K=$2; shift 2
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_${TAG}.log 2>&1; echo smoke=$? > gpurun_out/status_${TAG}.txt
if [ -n "$K" ]; then
  timeout 1500 python -m pytest tests -m gpu -x -q -k "$K" > gpurun_out/pytest_${TAG}.log 2>&1; echo pytest=$? >> gpurun_out/status_${TAG}.txt
fi
i=0
for e in "$@"; do
  env $e timeout 600 python bench.py --no-cpu-baseline ${BENCH_ARGS:-} > gpurun_out/bench_${TAG}_$i.log 2>&1
  echo "bench[$e]=$? $(tail -1 gpurun_out/bench_${TAG}_$i.log | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["ms_per_step"], {k: round(v["ms_per_step"],2) for k,v in d["roofline"]["phases"].items()}, d["e2e"]["ms_per_step"])' 2>&1)" >> gpurun_out/status_${TAG}.txt
  i=$((i+1))
done
cat gpurun_out/status_${TAG}.txt
