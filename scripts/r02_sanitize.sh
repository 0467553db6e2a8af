#!/bin/bash
# compute-sanitizer over the round-2 kernels (small grids): memcheck, racecheck, synccheck
OUT=gpurun_out/r02p; mkdir -p $OUT
CS=/usr/local/cuda/bin/compute-sanitizer
cat > /tmp/san_cases.py <<'PY'
import sys, numpy as np, torch
sys.path.insert(0, ".")
import oracle, synth
import paper_conf_ppopp_chenlwbwmyzcy24_b200 as csx
cases = [("box3d125p", (20, 37, 70), "tc_tile", 0, 2), ("star3d19p", (20, 37, 70), "tc_tile", 0, 2),
         ("box3d343p", (20, 37, 70), "tc_tile", 0, 1), ("box2d9p", (131, 150), "direct", 4, 9),
         ("heat2d", (131, 150), "direct", 3, 7), ("box2d25p", (131, 150), "direct", 1, 3),
         ("box2d9p", (99, 140), "tc_s2r", 3, 7), ("box2d25p", (99, 140), "tc_s2r", 1, 3)]
worst = 0.0
for name, ext, eng, tf, T in cases:
    s = synth.SHAPES[name]
    w = synth.random_weights(name)
    u0 = synth.grid(ext, seed=5)
    for bc in ("fixed", "periodic"):
        p = csx.Plan(ext, w, shape=s.kind, bc=bc, fuse_steps=tf, engine=eng)
        p.set_max_ctas(3)
        d_in = torch.from_numpy(u0).cuda(); d_out = torch.empty_like(d_in)
        p.run(d_in, d_out, T); torch.cuda.synchronize()
        ref = oracle.run(u0, w, bc, T)
        worst = max(worst, float(np.max(np.abs(d_out.cpu().numpy() - ref)) / np.max(np.abs(ref))))
        p.close()
print("worst rel err", worst)
PY
for tool in memcheck racecheck synccheck; do
  timeout 1500 $CS --tool $tool --print-limit 20 python /tmp/san_cases.py > $OUT/${tool}.txt 2>&1
  echo "rc=$?" >> $OUT/${tool}.txt
done
