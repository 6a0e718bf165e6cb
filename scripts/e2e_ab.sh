#!/bin/bash
for c in 2 1; do
  STG_E2E_COPY_STREAMS=$c timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench_e2e_cs$c.log 2>&1
  python -c "import json;d=json.loads([l for l in open('gpurun_out/bench_e2e_cs$c.log') if l.startswith('{')][-1]);print('copy_streams=$c', d['ms_per_step'], d['e2e'])" >> gpurun_out/e2e_ab.txt 2>&1
done
