b() { timeout 300 python bench.py --config $1 --ib $2 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e 2>&1 | tail -1 | python -c "
import json,sys
t=sys.stdin.read()
try:
  d=json.loads(t); print('ib', d['config']['ib'], d['config']['workload'], d['value'], d['ms_per_step'], d['roofline']['frac'])
except Exception as e: print('FAILED', t[-500:])"; }
for cfg in "4 8" "2 8" "4 16" "1 8"; do set -- $cfg; echo "split=$1 wlook=$2"; TQR_PANEL_SPLIT=$1 TQR_W_LOOK=$2 b C2 32; done
echo "C3/C5 ib16 w16"; b C3 16; b C5 16
