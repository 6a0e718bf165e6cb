# sensitivity of the Σ AᵀB reductions (dL, dW) to the TMA ring depth
for kb in 100 150 220; do
  STG_ATB_SMEM_KB=$kb timeout 500 python bench.py --no-cpu-baseline --no-e2e --naive > gpurun_out/bench_atb.log 2>&1
  tail -1 gpurun_out/bench_atb.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); p=d['phases_ms_per_step']; print('$kb KB', round(d['ms_per_step'],1), 'dl', round(p['dl'],2), 'dw', round(p['dw'],2))"
done
