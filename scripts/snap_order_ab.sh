#!/bin/bash
# forward snapshot-build placement A/B: after conv(t) (default) vs after conv(t-1)
for v in 1 0 1 0; do
  STG_SNAP_AFTER_CONV=$v timeout 900 python bench.py --no-e2e --no-cpu-baseline > gpurun_out/bench_sac$v.log 2>&1
  python -c "import json;d=json.loads([l for l in open('gpurun_out/bench_sac$v.log') if l.startswith('{')][-1]);r=d['roofline'];print('after_conv=$v', d['ms_per_step'], d['single_stream_ms_per_step'], round(r['avg_fwd_ms'],4), round(r['avg_bwd_ms'],4), round(r['frac'],4))" >> gpurun_out/snap_order_ab.txt
done
