#!/usr/bin/env bash
# a8 at human scale: cfg5 (1.25 G reads of 100 bp, 124.8 GB of ASCII in page-locked host
# memory, a 1.1 TB table set) through bench.py's streaming mode on one B200.
#   scripts/gpu_cfg5.sh TAG [extra bench args]
set -u
TAG=${1:-cfg5}
shift 1 2>/dev/null
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_${TAG}.log 2>&1
( while true; do date +%T; free -g | sed -n 2p; nvidia-smi --query-gpu=memory.used,clocks.sm --format=csv,noheader; sleep 10; done ) > gpurun_out/mon_${TAG}.txt 2>&1 &
MON=$!
if [ -n "${SMALL:-}" ]; then
timeout 900 python bench.py --config cfg5 --n 50000000 --steps 2 --warmup 3 "$@" > gpurun_out/bench_${TAG}_small.log 2>&1; echo small=$? >> gpurun_out/status_${TAG}.txt
fi
timeout ${CFG5_TIMEOUT:-2400} python bench.py --config cfg5 --steps 2 --warmup 3 "$@" > gpurun_out/bench_${TAG}.log 2>&1; echo cfg5=$? >> gpurun_out/status_${TAG}.txt
kill $MON
