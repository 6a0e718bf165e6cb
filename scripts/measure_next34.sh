timeout 300 python scripts/agg_weighted_probe.py > gpurun_out/weighted_probe.jsonl 2>&1
timeout 500 python bench.py --no-cpu-baseline --no-e2e --naive > gpurun_out/bench_naive.log 2>&1
timeout 500 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/bench_ondemand.log 2>&1
timeout 300 python bench.py --config C4 --no-cpu-baseline --no-e2e --naive > gpurun_out/bench_c4_naive.log 2>&1
timeout 300 python bench.py --config C4 --no-cpu-baseline --no-e2e > gpurun_out/bench_c4_ondemand.log 2>&1
cat gpurun_out/weighted_probe.jsonl
for f in bench_naive bench_ondemand bench_c4_naive bench_c4_ondemand; do tail -1 gpurun_out/$f.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$f', d['ms_per_step'], d['timesteps_per_s'], d['graph_memory_bytes'])"; done
