#!/bin/bash
# quick bench summary lines for a list of configs (GPU box)
for c in "$@"; do
  timeout 300 python bench.py --config $c --steps 2 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | python -c "
import json,sys
t=sys.stdin.read()
try:
    d=json.loads(t); print(d['config']['workload'], 'GF/s', d['value'], 'ms', d['ms_per_step'], 'upd_TF', d['roofline']['achieved'], 'share', d['roofline']['share_of_step'], 'panel', d['panel'], 'clk', d['clocks']['sm_mhz'], d['clocks']['reasons'])
except Exception as e: print('FAILED', t[-2000:])
"
done
