"""Ad-hoc parity of the k_tile3d_tb2 geometries (CSX_TB_GEOM) against the oracle: Heat-3D and a
box, both boundaries, ragged tiles, several z chunks, persistent grid capped so CTAs wrap."""
import os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle, synth
import paper_conf_ppopp_chenlwbwmyzcy24_b200 as csx
worst = 0.0
for name, ext in (("heat3d", (70, 61, 150)), ("box3d27p", (40, 57, 130)), ("heat3d", (9, 29, 65))):
    s = synth.SHAPES[name]; w = synth.random_weights(name); u0 = synth.grid(ext, seed=5)
    for bc in ("fixed", "periodic"):
        for cap in (3, 0):
            p = csx.Plan(ext, w, shape=s.kind, bc=bc, fuse_steps=2, engine="tc_tile")
            if cap: p.set_max_ctas(cap)
            d_in = torch.from_numpy(u0).cuda(); d_out = torch.empty_like(d_in)
            p.run(d_in, d_out, 5); torch.cuda.synchronize()
            ref = oracle.run(u0, w, bc, 5)
            e = float(np.max(np.abs(d_out.cpu().numpy() - ref)) / np.max(np.abs(ref))); p.close()
            worst = max(worst, e)
            assert e <= 1e-12, (name, ext, bc, cap, e)
print("tb2 geom", os.environ.get("CSX_TB_GEOM", "default"), "worst rel err", worst)
