#!/usr/bin/env bash
# Final round evidence that fits gpurun's 64 MiB return: bench line, a pytest selection,
# the launch list and ncu --set full of the scatter and join kernels.
#   scripts/gpu_final.sh TAG "pytest -k expr"
set -u
TAG=$1; K=${2:-}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_${TAG}.log 2>&1; echo smoke=$? > gpurun_out/status_${TAG}.txt
timeout 900 python bench.py > gpurun_out/bench_${TAG}.log 2>&1; echo bench=$? >> gpurun_out/status_${TAG}.txt
if [ -n "$K" ]; then
  timeout 1800 python -m pytest tests -m gpu -x -q -k "$K" > gpurun_out/pytest_${TAG}.log 2>&1; echo pytest=$? >> gpurun_out/status_${TAG}.txt
fi
bash scripts/profile_round.sh ${TAG} cfg3 scatter_table bucket_join > /dev/null 2>&1; echo profile=$? >> gpurun_out/status_${TAG}.txt
du -sh gpurun_out
cat gpurun_out/status_${TAG}.txt
