#!/bin/bash
# A/B an environment switch on the GPU box: scripts/ab_env.sh VAR "v1 v2" cfg1 cfg2 ... [-- extra bench args]
# prints workload, VAR=value, GSt/s, roofline frac for each combination.
VAR=$1; VALS=$2; shift 2
CFGS=(); EXTRA=()
while [ $# -gt 0 ]; do
  if [ "$1" == "--" ]; then shift; EXTRA=("$@"); break; fi
  CFGS+=("$1"); shift
done
for cfg in "${CFGS[@]}"; do
  for v in $VALS; do
    line=$(env $VAR=$v timeout 600 python bench.py --config $cfg --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator "${EXTRA[@]}" 2>/dev/null | tail -1)
    python -c "
import json,sys
try:
    d=json.loads(sys.argv[1]); r=d.get('roofline') or {}
    print(f'{sys.argv[2]:18s} $VAR=$v {d[\"value\"]:9.1f} {d[\"unit\"]} frac={r.get(\"frac\",0):.3f} ms/step={d[\"ms_per_step\"]:.3f}')
except Exception as e:
    print(sys.argv[2], '$VAR=$v', 'ERROR', sys.argv[1][:200])
" "$line" "$cfg"
  done
done
