for mode in 1 0; do
  for c in C3 C1; do
    TG_GRAPH_LOOP=$mode timeout 600 python bench.py --config $c --steps 12 --warmup 3 --no-cpu-baseline --no-e2e > /tmp/b.json 2>/dev/null
    python -c "
import json; d=json.load(open('/tmp/b.json')); print('graph_loop=$mode', '$c', round(d['value'],1), d['step_ms'])"
  done
done
