import sys, os, torch
sys.path.insert(0, ".")
import synth, bench
import paper_conf_ppopp_chenlwbwmyzcy24_b200 as csx
cfg = sys.argv[1] if len(sys.argv) > 1 else "heat3d_512"
shape, ext, T, bc, tf = bench.CONFIGS[cfg]
s = synth.SHAPES[shape]
p = csx.Plan(ext, synth.physical_weights(shape), shape=s.kind, bc=bc, engine="tc_tile")
if os.environ.get("CTAS"): p.set_max_ctas(int(os.environ["CTAS"]))
d_in = synth.grid_torch(ext, "cuda"); d_out = torch.empty_like(d_in)
p.run(d_in, d_out, 6); torch.cuda.synchronize()
e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
e0.record(); p.run(d_in, d_out, 10); e1.record(); torch.cuda.synchronize()
print(cfg, "lockstep", os.environ.get("CSX_LOCKSTEP"), "ms/step", e0.elapsed_time(e1) / 10, "GSt/s", 10 * d_in.numel() / e0.elapsed_time(e1) / 1e6)
