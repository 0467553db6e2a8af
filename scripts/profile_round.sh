#!/bin/bash
# On the GPU box: launch list + ncu captures (make_profiles.sh), summarised to text on the box
# (the .ncu-rep files are too large to bring back), then one bench line per config and engine.
#   bash scripts/profile_round.sh r01 <configs...>
TAG=$1; shift
bash scripts/make_profiles.sh $TAG > /dev/null 2>&1
cp profiles/traffic.json gpurun_out/$TAG/traffic.json 2>/dev/null
for rep in gpurun_out/$TAG/prof_*.ncu-rep; do
  name=$(basename $rep .ncu-rep); name=${name#prof_}
  key=$(python - "$name" <<'PY'
import sys
n = sys.argv[1]
cfg = {"box2d9p": "box2d9p_10240", "box2d49p": "box2d49p_10240", "box2d49p_tf2": "box2d49p_10240_tf2",
       "box3d27p": "box3d27p_512", "heat3d": "heat3d_512", "heat1d": "heat1d_10240000",
       "1d5p": "1d5p_10240000"}
base, eng = n.rsplit("_tc_", 1) if "_tc_" in n else n.rsplit("_", 1)
eng = ("tc_" + eng) if "_tc_" in n else eng
print(f"{cfg.get(base, base)}:{eng}")
PY
)
  echo "### $(basename $rep)" >> gpurun_out/$TAG/ncu_summaries.md
  python scripts/ncu_summary.py $rep --key $key --traffic gpurun_out/$TAG/traffic.json >> gpurun_out/$TAG/ncu_summaries.md 2>&1
  python scripts/ncu_brief.py $rep > gpurun_out/$TAG/brief_$name.txt 2>&1
done
mkdir -p /tmp/reps && mv gpurun_out/$TAG/*.ncu-rep /tmp/reps/ 2>/dev/null
[ $# -gt 0 ] && bash scripts/bench_all.sh "$@"
ls -la gpurun_out/$TAG
