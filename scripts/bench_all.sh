#!/bin/bash
# On the GPU box: one bench line per BASELINE config and engine -> gpurun_out/bench_all.jsonl
OUT=gpurun_out/bench_all.jsonl
: > $OUT
for cfg in "$@"; do
  for eng in auto tc_s2r direct; do
    timeout 600 python bench.py --config $cfg --engine $eng --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator >> $OUT 2>>gpurun_out/bench_all.err || echo "{\"config\": \"$cfg\", \"engine\": \"$eng\", \"error\": true}" >> $OUT
  done
done
python - <<'PY'
import json
for line in open("gpurun_out/bench_all.jsonl"):
    try:
        d = json.loads(line)
    except Exception:
        continue
    if "error" in d:
        print(d); continue
    r = d.get("roofline") or {}
    print(f'{d["config"]["workload"]:18s} {d["config"]["engine"]:8s} nk={d["config"]["nk"]:2d} {d["value"]:9.1f} GSt/s  {r.get("bound","-"):6s} frac={r.get("frac",0):.3f}  tc_share={r.get("tc_share_of_step",0) or 0:.3f}')
PY
