#!/usr/bin/env bash
# Box facts + a baseline bench of HEAD (1 GPU).
set -u
mkdir -p gpurun_out
{ nproc; lscpu | grep -E 'Model name|Socket|Thread|Core'; free -g; nvidia-smi --query-gpu=name,memory.total,clocks.max.sm --format=csv; nvidia-smi topo -m | head -5; } > gpurun_out/probe_box.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/probe_build.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/probe_bench.log 2>&1; echo bench=$? >> gpurun_out/probe_box.txt
