#!/bin/bash
timeout 600 python -m pytest tests/test_gpu_tgcn.py tests/test_gpu_dtdg.py -m gpu -x -q > gpurun_out/pytest_graph.log 2>&1; echo rc=$? >> gpurun_out/pytest_graph.log
rm -f gpurun_out/graphs_ab.txt
for c in C4 C5; do
  for gph in 1 0; do
    timeout 600 python bench.py --config $c --graphs $gph --no-e2e --no-cpu-baseline > gpurun_out/bench_${c}_g$gph.log 2>&1
    python -c "import json;d=json.loads([l for l in open('gpurun_out/bench_${c}_g$gph.log') if l.startswith('{')][-1]);print('$c graphs=$gph', d['ms_per_step'], d['config']['cuda_graph'], d['gpu_launches'], d['roofline']['frac'])" >> gpurun_out/graphs_ab.txt 2>&1
  done
done
