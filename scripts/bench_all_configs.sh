# one bench line per BASELINE.json config (C1-C3 static-temporal, C4/C5 DTDG); no e2e / cpu baseline
for c in C1 C2 C3 C4 C5; do
  timeout 600 python bench.py --config $c --no-cpu-baseline --no-e2e > gpurun_out/bench_$c.log 2>&1
  tail -1 gpurun_out/bench_$c.log >> gpurun_out/configs.jsonl
  tail -1 gpurun_out/bench_$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', round(d['ms_per_step'],2), 'ms/epoch', round(d['timesteps_per_s']), 'timesteps/s', '%.3g edges/s' % d['value'], d['config'].get('schedule'))"
done
