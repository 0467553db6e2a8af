#!/bin/bash
# On the GPU box: problem-size sweep (the paper's Fig 8 axes): 2D 256..5120
# step 256 (Box-2D9P, Heat-2D), 3D 64..1024 step 32 (Heat-3D, Box-3D27P), TC_TILE, own curve only.
# FROM3D / TO3D / SKIP2D narrow the run (e.g. FROM3D=544 SKIP2D=1 appends the large 3D sizes).
OUT=${OUT:-gpurun_out/size_sweep.jsonl}
[ -z "$APPEND" ] && : > $OUT
[ -z "$SKIP2D" ] && for n in $(seq ${STEP2D:-256} ${STEP2D:-256} 5120); do
  for sh in box2d9p heat2d; do
    python bench.py --shape $sh --grid $n,$n --T 100 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator >> $OUT 2>/dev/null
  done
done
for n in $(seq ${FROM3D:-64} ${STEP3D:-32} ${TO3D:-1024}); do
  for sh in heat3d box3d27p; do
    python bench.py --shape $sh --grid $n,$n,$n --T 50 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator >> $OUT 2>/dev/null
  done
done
OUT=$OUT python - <<'PY'
import json
import os
for line in open(os.environ.get("OUT", "gpurun_out/size_sweep.jsonl")):
    d = json.loads(line); c = d["config"]
    print(f'{c["workload"]} {"x".join(map(str, c["grid"])):16s} {d["value"]:8.1f} GSt/s  frac={(d.get("roofline") or {}).get("frac", 0):.3f}')
PY
