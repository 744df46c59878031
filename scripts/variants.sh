# Run bench.py under several environment variants (opt-in kernel paths), one JSON summary each.
# usage: bash scripts/variants.sh [workload] "ENV1=a ENV2=b" "ENV3=c" ...
wl=$1; shift
for v in "$@"; do
  env $v timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-extras --workload $wl 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().splitlines()[-1])
print('$v', round(d['value'],1), round(d['ms_per_step']*1e3,2), {k: round(v*1e3,2) for k,v in d['stages_ms'].items()})"
done
