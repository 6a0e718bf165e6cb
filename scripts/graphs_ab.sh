#!/bin/bash
for c in C4 C5; do
  for gph in 0 1; do
    timeout 900 python bench.py --config $c --graphs $gph --no-e2e --no-cpu-baseline > gpurun_out/bench_${c}_g$gph.log 2>&1
    python -c "import json;d=json.loads([l for l in open('gpurun_out/bench_${c}_g$gph.log') if l.startswith('{')][-1]);print('$c graphs=$gph', d['ms_per_step'], d['config']['cuda_graph'], d['gpu_launches'], d['roofline']['frac'])" >> gpurun_out/graphs_ab.txt 2>&1
  done
done
