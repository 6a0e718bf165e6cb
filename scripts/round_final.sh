# Round-end evidence on one B200: GPU tests, smoke, default bench (with e2e + cpu
# baseline), steady-state launch list, ncu --set full of the hot kernels.
set -x
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_default.log 2>&1
bash scripts/seq_launches.sh
python scripts/steady_summary.py gpurun_out/launches_seq.csv > gpurun_out/steady.txt 2>&1
bash scripts/ncu_capture.sh
python scripts/ncu_extract.py > gpurun_out/ncu_full.json 2>&1
tail -3 gpurun_out/pytest_gpu.log; tail -1 gpurun_out/smoke.log; tail -1 gpurun_out/bench_default.log | cut -c1-300; head -12 gpurun_out/steady.txt
