"""One csx_run of a bench configuration (no graph, no timing): the process ncu attaches to for
the DMMA / DRAM counters of the dominant kernel (scripts/dmma_counters.py).  Prints the plan
info (incl. the planner's DMMA count per main pass) as one JSON line on stdout."""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import synth  # noqa: E402
import paper_conf_ppopp_chenlwbwmyzcy24_b200 as csx  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", required=True)
ap.add_argument("--engine", default="auto")
ap.add_argument("--T", type=int, default=None)
ap.add_argument("--fuse", type=int, default=None)
args = ap.parse_args()
shape, ext, T, bc, tf = bench.CONFIGS[args.config]
T = args.T or T
s = synth.SHAPES[shape]
w = synth.physical_weights(shape)
p = csx.Plan(ext, w, shape=s.kind, bc=bc, fuse_steps=tf if args.fuse is None else args.fuse, engine=args.engine)
d_in = synth.grid_torch(ext, "cuda")
d_out = torch.empty_like(d_in)
p.run(d_in, d_out, T)
torch.cuda.synchronize()
info = p.info()
info["points"] = int(np.prod(ext))
info["T"] = T
print(json.dumps(info), flush=True)
p.close()
