#!/usr/bin/env bash
# Round evidence on one B200: smoke, the full GPU suite, the default bench (with the CPU
# baseline), then the launch list and ncu --set full captures (scripts/profile_round.sh).
#   scripts/gpu_full.sh TAG
set -u
TAG=${1:-r01}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_${TAG}.log 2>&1; echo smoke=$? > gpurun_out/status_${TAG}.txt
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_${TAG}.log 2>&1; echo pytest=$? >> gpurun_out/status_${TAG}.txt
timeout 900 python bench.py > gpurun_out/bench_${TAG}.log 2>&1; echo bench=$? >> gpurun_out/status_${TAG}.txt
bash scripts/profile_round.sh ${TAG} cfg3 > /dev/null 2>&1; echo profile=$? >> gpurun_out/status_${TAG}.txt
cat gpurun_out/status_${TAG}.txt
