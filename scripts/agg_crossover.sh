# strategy 1 (pipelined items) vs 2 (edge stream) across graph sizes and widths
for cw in "C1 48" "C2 96" "C2 1536" "C3 96" "C3 1536" "C4 96" "C5s 96"; do
  set -- $cw
  timeout 300 python scripts/agg_sweep.py --config $1 --W $2 --only "s" 2>/dev/null | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l)
    if d['name'] in ('s1','s2 d16 minb3'): print('$1', d['E'], d['W'], d['name'], d['fwd']['ms'], d['bwd']['ms'])
"
done
