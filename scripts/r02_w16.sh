#!/bin/bash
OUT=gpurun_out/r02w16; mkdir -p $OUT
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator"
for c in star3d13p_512 star3d19p_512; do for w in 0 1; do
  echo "$c w16=$w $(CSX_TILE3D_W16=$w timeout 300 $B --config $c 2>/dev/null)" >> $OUT/ab.txt; done; done
for w in 0 1; do echo "heat3d_tf1 w16=$w $(CSX_TILE3D_W16=$w timeout 300 $B --config heat3d_512 --fuse 1 2>/dev/null)" >> $OUT/ab.txt; done
cat > /tmp/w16_parity.py <<'PY'
import sys, numpy as np, torch
sys.path.insert(0, ".")
import oracle, synth
import paper_conf_ppopp_chenlwbwmyzcy24_b200 as csx
worst = 0.0
for name, T in (("heat3d", 3), ("star3d13p", 2), ("star3d19p", 2)):
    s = synth.SHAPES[name]; w = synth.random_weights(name)
    for ext in ((45, 37, 70), (40, 70, 130)):
        u0 = synth.grid(ext, seed=9)
        for bc in ("fixed", "periodic"):
            for cap in (3, 0):
                p = csx.Plan(ext, w, shape=s.kind, bc=bc, fuse_steps=1, engine="tc_tile")
                if cap: p.set_max_ctas(cap)
                d_in = torch.from_numpy(u0).cuda(); d_out = torch.empty_like(d_in)
                p.run(d_in, d_out, T); torch.cuda.synchronize()
                ref = oracle.run(u0, w, bc, T)
                e = float(np.max(np.abs(d_out.cpu().numpy() - ref)) / np.max(np.abs(ref))); p.close()
                worst = max(worst, e); assert e <= 1e-12, (name, ext, bc, cap, e)
print("w16 worst rel err", worst)
PY
CSX_TILE3D_W16=1 timeout 300 python /tmp/w16_parity.py > $OUT/parity.txt 2>&1
