#!/bin/bash
# Round-end evidence on one B200: GPU tests, smoke, default bench (with e2e + cpu baseline),
# aggregate-first and sharded-mode (N=1) benches, steady-state launch list, snapshot step
# timings + launch list (the ncu --set full captures: scripts/round_ncu.sh).
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_default.log 2>&1
timeout 900 python bench.py --order aggregate-first --no-e2e --no-cpu-baseline > gpurun_out/bench_aggfirst.log 2>&1
timeout 900 python bench.py --mode peer --no-e2e --no-cpu-baseline > gpurun_out/bench_peer_n1.log 2>&1
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_reference.log 2>&1
bash scripts/seq_launches.sh
python scripts/steady_summary.py gpurun_out/launches_seq.csv > gpurun_out/steady.txt 2>&1
timeout 300 python scripts/snapshot_probe2.py > gpurun_out/snapshot_probe2.log 2>&1
PROBE_NCU=1 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/snapshot_launches.csv python scripts/snapshot_probe2.py > gpurun_out/ncu_snap.log 2>&1
python scripts/launch_summary.py gpurun_out/snapshot_launches.csv > gpurun_out/snapshot_launches.txt 2>&1
tail -3 gpurun_out/pytest_gpu.log; tail -1 gpurun_out/smoke.log; tail -1 gpurun_out/bench_default.log | cut -c1-300; head -12 gpurun_out/steady.txt
