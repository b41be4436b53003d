# one bench line, summarised: bash scripts/qb.sh <bench.py args...>
timeout 600 python bench.py --no-e2e --no-cpu "$@" 2>/dev/null | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read())
pk={k:(round(v['achieved']) if v.get('achieved') is not None else None) for k,v in d.get('per_kernel',{}).items()}
print('$*', d['value'], d['unit'], 'sm', d['clocks']['sm_mhz'], 'frac', d['roofline']['frac'])"
