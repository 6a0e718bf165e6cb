# parallel fixed-order partial sums (k_tc_sum_parts2): GPU tests, 2 bench runs, launch list
timeout 900 python -m pytest tests/test_gpu_tc.py tests/test_gpu_tgcn.py tests/test_gpu_dtdg.py tests/test_gpu_static.py -m gpu -x -q > gpurun_out/pytest_tc.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_tc.log
tail -3 gpurun_out/pytest_tc.log
for c in 1 2; do
  timeout 500 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/bench_sum2_$c.log 2>&1
  tail -1 gpurun_out/bench_sum2_$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); p=d['phases_ms_per_step']; print(round(d['ms_per_step'],1), {k: round(v,2) for k,v in p.items()}, round(d['roofline']['frac'],3))"
done
bash scripts/seq_launches.sh
python scripts/steady_summary.py gpurun_out/launches_seq.csv > gpurun_out/steady.txt 2>&1
grep -E "total|sum_parts|atb2" gpurun_out/steady.txt
