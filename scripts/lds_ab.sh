# explicit ld.shared in the Σ AᵀB converters and GRU raw-tile reads (was generic LD.E): tests + 2 bench runs
timeout 900 python -m pytest tests/test_gpu_tc.py tests/test_gpu_tgcn.py tests/test_gpu_dtdg.py -m gpu -x -q > gpurun_out/pytest_tc.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_tc.log
tail -3 gpurun_out/pytest_tc.log
for c in 1 2; do
  timeout 500 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/bench_lds_$c.log 2>&1
  tail -1 gpurun_out/bench_lds_$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); p=d['phases_ms_per_step']; print(round(d['ms_per_step'],1), {k: round(v,2) for k,v in p.items()}, round(d['roofline']['frac'],3))"
done
