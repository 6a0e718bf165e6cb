# ping-pong GRU forward (k_tc_gru_fwd3) vs k_tc_gru_fwd2: GPU tests + C5 bench A/B
timeout 900 python -m pytest tests/test_gpu_tc.py tests/test_gpu_tgcn.py tests/test_gpu_dtdg.py tests/test_gpu_static.py -m gpu -x -q > gpurun_out/pytest_tc.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_tc.log
tail -3 gpurun_out/pytest_tc.log
for c in 0 1 0 1; do
  STG_GRU_FWD3=$c timeout 500 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/bench_fwd3_$c.log 2>&1
  tail -1 gpurun_out/bench_fwd3_$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); p=d['phases_ms_per_step']; print('fwd3=$c', round(d['ms_per_step'],1), 'gru_fwd', round(p['gru_fwd'],2), 'gru_bwd', round(p['gru_bwd'],2), round(d['roofline']['frac'],3))"
done
