#!/bin/bash
# Epoch time of the C5 bench under scheduling knobs (pipelined sequence driver).
set -u
run() {  # name, env...
  local name=$1; shift
  env "$@" python bench.py --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > gpurun_out/sweep_$name.json 2>/dev/null
  python - "$name" <<'PY'
import json, sys
n = sys.argv[1]
d = json.loads(open("gpurun_out/sweep_%s.json" % n).read().strip().splitlines()[-1])
print(json.dumps({"name": n, "ms_per_step": round(d["ms_per_step"], 2), "Gedges_s": round(d["value"] / 1e9, 3),
                  "phases": {k: round(v, 1) for k, v in d["phases_ms_per_step"].items()}}))
PY
}
for cfg in "$@"; do
  name=${cfg%%:*}; envs=${cfg#*:}
  run "$name" $envs
done
