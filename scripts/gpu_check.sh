#!/usr/bin/env bash
# GPU check: build, smoke, pytest -m gpu (optionally with a -m/-k filter), bench (1 GPU).
#   scripts/gpu_check.sh TAG ["pytest marker expr"]      e.g. scripts/gpu_check.sh x "gpu and not slow"
set -u
TAG=${1:-chk}
M=${2:-gpu}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_${TAG}.log 2>&1; echo smoke=$? > gpurun_out/status_${TAG}.txt
timeout 1500 python -m pytest tests -m "$M" -x -q > gpurun_out/pytest_${TAG}.log 2>&1; echo pytest=$? >> gpurun_out/status_${TAG}.txt
timeout 900 python bench.py ${BENCH_ARGS:-} > gpurun_out/bench_${TAG}.log 2>&1; echo bench=$? >> gpurun_out/status_${TAG}.txt
