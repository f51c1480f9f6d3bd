#!/usr/bin/env bash
# Interleaved A/B of environment settings on one B200: bench.py (cfg3, no CPU baseline) under
# each setting in turn, REPS times.  Prints one summary line per run.
#   scripts/gpu_ab_env.sh TAG REPS "A=env settings" "B=env settings" ...
set -u
TAG=$1; REPS=$2; shift 2
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_${TAG}.log 2>&1
for r in $(seq 1 $REPS); do
  for spec in "$@"; do
    name=${spec%%=*}; envs=${spec#*=}
    env $envs timeout 600 python bench.py --no-cpu-baseline --steps 5 --warmup 3 ${BENCH_ARGS:-} > gpurun_out/ab_${TAG}_${name}_${r}.log 2>&1
    python - "$name" "$r" gpurun_out/ab_${TAG}_${name}_${r}.log <<'PY' >> gpurun_out/ab_${TAG}.txt
import json, sys
name, r, path = sys.argv[1:4]
try:
    d = json.loads([l for l in open(path) if l.startswith("{")][-1])
    ph = d["roofline"]["phases"]
    print(name, r, "step %.2f" % d["ms_per_step"], "e2e %.2f" % d["e2e"]["ms_per_step"],
          " ".join("%s %.2f" % (k.split("_")[0], v["ms_per_step"]) for k, v in ph.items()))
except Exception as e:
    print(name, r, "FAILED", e, open(path).read()[-500:].replace("\n", " | "))
PY
  done
done
cat gpurun_out/ab_${TAG}.txt
