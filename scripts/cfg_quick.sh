#!/bin/bash
rm -f gpurun_out/configs.jsonl
for c in C1 C4 C5; do
  timeout 600 python bench.py --config $c --no-cpu-baseline --no-e2e > gpurun_out/bench_$c.log 2>&1
  python -c "import json;d=json.loads([l for l in open('gpurun_out/bench_$c.log') if l.startswith('{')][-1]);print('$c', d['ms_per_step'], d['config']['cuda_graph'], d['timesteps_per_s'], d['roofline']['frac'], d['roofline']['timing'][:60])" >> gpurun_out/cfg_quick.txt 2>&1
done
