timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_all.log 2>&1; tail -2 gpurun_out/pytest_all.log
timeout 500 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/bench_q.log 2>&1
tail -1 gpurun_out/bench_q.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C5', d['ms_per_step'], {k:round(v,1) for k,v in d['phases_ms_per_step'].items()})"
timeout 300 python bench.py --config C4 --no-cpu-baseline --no-e2e > gpurun_out/bench_q4.log 2>&1
tail -1 gpurun_out/bench_q4.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C4', d['ms_per_step'])"
bash scripts/seq_launches.sh; python scripts/steady_summary.py gpurun_out/launches_seq.csv > gpurun_out/steady.txt; head -30 gpurun_out/steady.txt
