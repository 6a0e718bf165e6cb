#!/bin/bash
# Snapshot-builder check on one B200: the snapshot / schedule tests, step timings, launch list.
set -x
timeout 1200 python -m pytest tests/test_gpu_dtdg.py tests/test_gpu_static.py tests/test_gpu_shard.py tests/test_gpu_naive.py tests/test_gpu_fullsize.py -m gpu -x -q > gpurun_out/pytest_snap.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_snap.log
timeout 300 python scripts/snapshot_probe2.py > gpurun_out/snapshot_probe2.log 2>&1
PROBE_NCU=1 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/snapshot_launches.csv python scripts/snapshot_probe2.py > gpurun_out/ncu_snap.log 2>&1
python scripts/launch_summary.py gpurun_out/snapshot_launches.csv > gpurun_out/snapshot_launches.txt 2>&1
tail -3 gpurun_out/pytest_snap.log; tail -2 gpurun_out/snapshot_probe2.log; grep -E 'k_merge3|k_touch3|k_rowscan|k_ids|k_items' gpurun_out/snapshot_launches.txt
