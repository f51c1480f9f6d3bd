#!/usr/bin/env bash
# GPU check: build, smoke, pytest (marker expr, no -x so every failure shows), bench (1 GPU).
#   scripts/gpu_check.sh TAG ["pytest marker expr"] [pytest args...]
set -u
TAG=${1:-chk}
M=${2:-gpu}
shift 2 2>/dev/null
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_${TAG}.log 2>&1; echo smoke=$? > gpurun_out/status_${TAG}.txt
timeout ${PYTEST_TIMEOUT:-2400} python -m pytest tests -m "$M" -q -rf --durations=15 --timeout=${TEST_TIMEOUT:-900} "$@" > gpurun_out/pytest_${TAG}.log 2>&1; echo pytest=$? >> gpurun_out/status_${TAG}.txt
if [ -z "${NO_BENCH:-}" ]; then
timeout 900 python bench.py ${BENCH_ARGS:-} > gpurun_out/bench_${TAG}.log 2>&1; echo bench=$? >> gpurun_out/status_${TAG}.txt
fi
