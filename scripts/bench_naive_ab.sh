# Table III analogue on C5 / C4: on-demand snapshots (default) vs NaiveGraph (STG_NAIVE)
for c in C5 C4; do
  for m in "" "--naive"; do
    timeout 500 python bench.py --config $c --no-cpu-baseline --no-e2e $m > gpurun_out/bench_nv.log 2>&1
    tail -1 gpurun_out/bench_nv.log >> gpurun_out/table3.jsonl
    tail -1 gpurun_out/bench_nv.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c $m', d['ms_per_step'], d['graph_memory_bytes'])"
  done
done
