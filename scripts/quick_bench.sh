# value, clock and per-kernel achieved of bench.py lines for the given configs
# (no e2e / cpu legs): bash scripts/quick_bench.sh bb vt lm
for c in "$@"; do
  timeout 600 python bench.py --config $c --no-e2e --no-cpu 2>/dev/null | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read())
pk={k:(round(v['achieved']) if v.get('achieved') is not None else None) for k,v in d.get('per_kernel',{}).items()}
print('$c', d['value'], d['unit'], 'sm', d['clocks']['sm_mhz'], 'frac', d['roofline']['frac'], pk)"
done
