# A/B of the Σ AᵀB reductions (k_tc_atb2): dL reduction with 2 CTAs/SM x (2 hi stages + 1 lo slot) vs 1 CTA x (4 + 2)
timeout 900 python -m pytest tests/test_gpu_tc.py tests/test_gpu_tgcn.py -m gpu -x -q > gpurun_out/pytest_tc.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_tc.log
tail -3 gpurun_out/pytest_tc.log
for c in 0 1 0 1; do
  STG_ATB_L1=$c timeout 500 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/bench_atb_l1_$c.log 2>&1
  tail -1 gpurun_out/bench_atb_l1_$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); p=d['phases_ms_per_step']; print('l1 $c', round(d['ms_per_step'],1), 'dl', round(p['dl'],2), 'dw', round(p['dw'],2), round(d['roofline']['frac'],3))"
done
