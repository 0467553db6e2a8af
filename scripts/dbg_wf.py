import sys, numpy as np, torch
sys.path.insert(0, '.')
import oracle, synth
import paper_conf_ppopp_chenlwbwmyzcy24_b200 as csx
for (R, tf, ext, bc, T) in [(1, 1, (131, 150), "fixed", 1), (1, 1, (131, 150), "periodic", 1), (1, 3, (131, 150), "periodic", 3),
                            (1, 1, (300, 260), "periodic", 1)]:
    w = synth.random_signed_weights(2, R, seed=40 + R)
    u0 = synth.grid(ext, seed=41)
    p = csx.Plan(u0.shape, w, shape="box", bc=bc, fuse_steps=tf, engine="direct")
    d_in = torch.from_numpy(u0).cuda()
    d_out = torch.full_like(d_in, float("nan"))
    p.run(d_in, d_out, T)
    torch.cuda.synchronize()
    got = d_out.cpu().numpy()
    ref = oracle.run(u0, w, bc, T)
    bad = ~(np.abs(got - ref) <= 1e-12)
    rows = np.where(bad.any(1))[0]; cols = np.where(bad.any(0))[0]
    print(R, tf, ext, bc, T, "bad", bad.sum(), "rows", rows[:10], rows[-5:], "cols", cols[:10], cols[-5:], "nan", np.isnan(got).sum())
    if bad.any():
        r, c = np.argwhere(bad)[0]
        print("  first bad", r, c, got[r, c], ref[r, c], "u0", u0[r, c])
        # is got equal to ref shifted?
        for dy in (-2, -1, 1, 2):
            print("  shift", dy, np.nanmax(np.abs(got[max(0,dy):ext[0]+min(0,dy)] - ref[max(0,-dy):ext[0]-max(0,dy)])))
    p.close()
