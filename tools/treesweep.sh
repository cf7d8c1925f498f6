#!/bin/bash
# sweep the elimination-tree domain length L (bench --tree) for the given configs (GPU box)
# usage: tools/treesweep.sh "C2 C3" "-1 2 4 8"
for c in $1; do
  for t in $2; do
    timeout 300 python bench.py --config $c --tree $t --steps 2 --warmup 3 --no-cpu-baseline --no-e2e $3 2>&1 | tail -1 | python -c "
import json,sys
t=sys.stdin.read()
try:
    d=json.loads(t); print('$c tree $t', 'GF/s', d['value'], 'ms', d['ms_per_step'], 'upd_TF', d['roofline']['achieved'], 'share', d['roofline']['share_of_step'], 'panel', d['panel'])
except Exception as e: print('$c tree $t FAILED', t[-1500:])
"
  done
done
