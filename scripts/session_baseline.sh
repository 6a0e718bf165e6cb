#!/bin/bash
# Session start check on one B200: GPU tests, smoke, default bench, peer-mode N=1 bench,
# snapshot step timings.
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1
timeout 900 python bench.py --no-e2e > gpurun_out/bench_default.log 2>&1
timeout 900 python bench.py --mode peer --no-e2e --no-cpu-baseline > gpurun_out/bench_peer_n1.log 2>&1
timeout 300 python scripts/snapshot_probe2.py > gpurun_out/snapshot_probe2.log 2>&1
tail -3 gpurun_out/pytest_gpu.log; tail -1 gpurun_out/smoke.log; tail -1 gpurun_out/bench_default.log | cut -c1-400; tail -1 gpurun_out/bench_peer_n1.log | cut -c1-400; tail -5 gpurun_out/snapshot_probe2.log
PROBE_NCU=1 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/snapshot_launches.csv python scripts/snapshot_probe2.py > gpurun_out/ncu_snap.log 2>&1
