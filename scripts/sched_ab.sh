#!/bin/bash
# pipelined-epoch schedule A/B on C5: default (aux compute stream + snapshot stream) vs
# STG_AUX_STREAM=0 (compute on the caller's stream, only the snapshot builds overlapped)
for v in 1 0 1 0; do
  STG_AUX_STREAM=$v timeout 900 python bench.py --no-e2e --no-cpu-baseline --steps 5 > gpurun_out/bench_aux$v.log 2>&1
  python -c "import json;d=json.loads([l for l in open('gpurun_out/bench_aux$v.log') if l.startswith('{')][-1]);print('aux=$v', d['ms_per_step'], d['single_stream_ms_per_step'])" >> gpurun_out/sched_ab.txt
done
