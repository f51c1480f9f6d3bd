#!/usr/bin/env bash
# compute-sanitizer over every kernel family (scripts/sanitize_driver.py), one tool per run.
set -u
TAG=${1:-r02}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_san_${TAG}.log 2>&1
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 99 --print-limit 50 \
      python scripts/sanitize_driver.py > gpurun_out/sanitize_${TAG}_${tool}.log 2>&1
  echo "$tool=$?" >> gpurun_out/status_san_${TAG}.txt
done
