#!/bin/bash
OUT=gpurun_out/r02s19; mkdir -p $OUT
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator"
for w in 0 2; do echo "star3d19p w16=$w $(CSX_TILE3D_W16=$w timeout 300 $B --config star3d19p_512 2>/dev/null)" >> $OUT/ab.txt; done
cat > /tmp/s19.py <<'PY'
import os, sys, numpy as np, torch
sys.path.insert(0, ".")
import oracle, synth
import paper_conf_ppopp_chenlwbwmyzcy24_b200 as csx
worst = 0.0
os.environ["CSX_TILE3D_W16"] = "2"
s = synth.SHAPES["star3d19p"]; w = synth.random_weights("star3d19p")
for ext in ((45, 37, 70), (40, 70, 130)):
    u0 = synth.grid(ext, seed=9)
    for bc in ("fixed", "periodic"):
        for cap in (3, 0):
            p = csx.Plan(ext, w, shape=s.kind, bc=bc, fuse_steps=1, engine="tc_tile")
            if cap: p.set_max_ctas(cap)
            d_in = torch.from_numpy(u0).cuda(); d_out = torch.empty_like(d_in)
            p.run(d_in, d_out, 2); torch.cuda.synchronize()
            ref = oracle.run(u0, w, bc, 2)
            e = float(np.max(np.abs(d_out.cpu().numpy() - ref)) / np.max(np.abs(ref))); p.close()
            worst = max(worst, e); assert e <= 1e-12, (ext, bc, cap, e)
print("s19 worst rel err", worst)
PY
timeout 300 python /tmp/s19.py > $OUT/parity.txt 2>&1
