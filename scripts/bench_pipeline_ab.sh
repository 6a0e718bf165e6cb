# A/B of the Algorithm-1 stream schedule on C5 (CUDA events, bench.py)
for cfg in "STG_AUX_STREAM=0" "STG_AUX_STREAM=1"; do
  env $cfg timeout 500 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/bench_ab.log 2>&1
  tail -1 gpurun_out/bench_ab.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg', d['ms_per_step'], {k:round(v,1) for k,v in d['phases_ms_per_step'].items()})"
  env $cfg timeout 500 python bench.py --no-cpu-baseline --no-e2e --naive > gpurun_out/bench_ab.log 2>&1
  tail -1 gpurun_out/bench_ab.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg naive', d['ms_per_step'])"
done
