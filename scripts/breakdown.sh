#!/bin/bash
# On the GPU box: the B200 analogue of the paper's Fig 6 breakdown on Box-2D9P 10240^2, T=100.
OUT=${OUT:-gpurun_out/breakdown.jsonl}
: > $OUT
CFG=${1:-box2d9p_10240}
python bench.py --config $CFG --engine direct --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator >> $OUT
for v in I II III IV V; do
  python bench.py --config $CFG --engine tc_s2r --s2r-variant $v --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator >> $OUT
done
python bench.py --config $CFG --engine tc_tile --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator >> $OUT
OUT=$OUT python - <<'PY'
import json
import os
for line in open(os.environ.get("OUT", "gpurun_out/breakdown.jsonl")):
    d = json.loads(line); c = d["config"]; r = d.get("roofline") or {}
    print(f'{c["workload"]:16s} {c["engine"]:8s} {str(c.get("s2r_variant")):5s} {d["value"]:8.1f} GSt/s  frac={r.get("frac", 0):.3f}')
PY
