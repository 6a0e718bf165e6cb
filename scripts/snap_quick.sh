#!/bin/bash
# quick snapshot check: DTDG tests (incl. merge edge cases) + step timings + launch list
timeout 900 python -m pytest tests/test_gpu_dtdg.py -m gpu -x -q > gpurun_out/pytest_snapq.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_snapq.log
timeout 300 python scripts/snapshot_probe2.py > gpurun_out/snapshot_probe2.log 2>&1
PROBE_NCU=1 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/snapshot_launches.csv python scripts/snapshot_probe2.py > gpurun_out/ncu_snap.log 2>&1
python scripts/launch_summary.py gpurun_out/snapshot_launches.csv > gpurun_out/snapshot_launches.txt 2>&1
