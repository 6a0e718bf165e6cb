#!/bin/bash
# snapshot quick check + default bench (no e2e / cpu baseline)
bash scripts/snap_quick.sh
timeout 900 python bench.py --no-e2e --no-cpu-baseline > gpurun_out/bench_default.log 2>&1
