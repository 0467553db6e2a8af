#!/usr/bin/env python
"""bench.py — FP64 GStencils/s of the csx hot path (ConvStencil on B200), one JSON line.

A "step" is one csx_run over one configuration: T base time steps of the stencil on the whole
grid (every §8(a) row: fused TC passes, remainder pass, FIXED band fix-up).  GStencils/s follows
Eq 16 (PAPER.md P.1896-1910): T * prod(N) / t / 1e9 with T in base steps (reading A5).

  python bench.py                          # N=1, Box-2D9P 10240^2, T=100 (BASELINE configs[1])
  torchrun --nproc-per-node N bench.py --gpus N   # weak-scaled slabs: (10240*N) x 10240 (config C5)
  python bench.py --impl reference         # the CPU oracle on the host cores (bounded sample)
  python bench.py --config box2d49p --engine direct ...

Timing: W untimed warm-up steps; K timed steps between barrier + cudaDeviceSynchronize, CUDA
events on the launching stream, max over ranks.  Inputs (839 MB per grid) are larger than the
126 MB L2, so no explicit flush is needed.  The dominant kernel's time is measured live by the
library's event hooks (csx_profile_*).
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synth  # noqa: E402

CONFIGS = {
    # name: (shape, extents, T, bc, fuse_steps)   — BASELINE.json configs
    "heat1d_1024": ("heat1d", (1024,), 16, "fixed", 0),                  # C1 (parity config)
    "box2d9p_10240": ("box2d9p", (10240, 10240), 100, "fixed", 0),       # C2 (headline)
    "star2d13p_10240": ("star2d13p", (10240, 10240), 100, "fixed", 0),   # C3
    "box2d49p_10240": ("box2d49p", (10240, 10240), 100, "fixed", 0),     # C3
    "heat3d_512": ("heat3d", (512, 512, 512), 50, "fixed", 0),           # C4
    "box3d27p_512": ("box3d27p", (512, 512, 512), 50, "fixed", 0),       # C4
    "heat1d_10240000": ("heat1d", (10240000,), 1000, "fixed", 0),        # extra (north-star list)
    "1d5p_10240000": ("1d5p", (10240000,), 1000, "fixed", 0),
    "heat2d_10240": ("heat2d", (10240, 10240), 100, "fixed", 0),
    "star2d9p_10240": ("star2d9p", (10240, 10240), 100, "fixed", 0),     # Table 3 extra shapes
    "box2d25p_10240": ("box2d25p", (10240, 10240), 100, "fixed", 0),
    # C3 "multi-step fused" as BASELINE.json words it: r = 3, Tf = 2 (nk = 13, reading A4/A7)
    "star2d13p_10240_tf2": ("star2d13p", (10240, 10240), 100, "fixed", 2),
    "box2d49p_10240_tf2": ("box2d49p", (10240, 10240), 100, "fixed", 2),
    # 1D well beyond the 126 MB L2 (819 MB per buffer), where HBM binds
    "heat1d_102400000": ("heat1d", (102400000,), 1000, "fixed", 0),
    "1d5p_102400000": ("1d5p", (102400000,), 1000, "fixed", 0),
    # general radius in 3D
    "box3d125p_512": ("box3d125p", (512, 512, 512), 50, "fixed", 0),
    "star3d13p_512": ("star3d13p", (512, 512, 512), 50, "fixed", 0),
    "box3d343p_512": ("box3d343p", (512, 512, 512), 10, "fixed", 0),
    "star3d19p_512": ("star3d19p", (512, 512, 512), 50, "fixed", 0),
}
DEFAULT = "box2d9p_10240"
METRIC = "FP64 GStencils/s"
UNIT = "GStencils/s"


def load_json(path):
    try:
        with open(path) as f:
            return json.load(f)
    except Exception:
        return None


def peaks():
    mp = load_json(os.path.join(ROOT, "MEASURED_PEAKS.json")) or {}
    fp = load_json(os.path.join(ROOT, "PEAKS_FP64.json")) or {}
    hbm = mp.get("hbm_gbs")
    hbm_src = "MEASURED_PEAKS.json hbm_gbs (measured copy)"
    if hbm is None:
        hbm, hbm_src = 6650.0, "fallback 6.65 TB/s (B200_PROFILING.md)"
    dmma = fp.get("dmma_tflops_sustained") or fp.get("dmma_tflops")
    dmma_src = "PEAKS_FP64.json dmma_tflops_sustained (on-box DMMA.8x8x4 microbenchmark, peaks/fp64_peaks.cu)"
    if dmma is None:
        dmma, dmma_src = 37.2, "nominal 148 SMs x 4 x 512 flop / 16 cyc x 1.965 GHz (no measurement found)"
    return float(hbm), hbm_src, float(dmma), dmma_src


class ClockSampler:
    """nvidia-smi clocks and throttle reasons, sampled every 20 ms by a reader thread that stamps
    each row with the host clock.  The sampler is started (and its first row awaited) before the
    timed region; mark() brackets the region on the host (the steps are enqueued inside it and it
    ends after the device synchronize, so it covers the device work).  summary() keeps the rows
    inside the region plus the one just before and just after it (a region shorter than the
    sampling period still gets the two samples that bracket it)."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index, period_ms=20):
        self.gpu = gpu_index
        self.period = period_ms
        self.proc = None
        self.rows = []  # (host monotonic time, [fields])
        self.t0 = self.t1 = None
        self.thread = None

    def _reader(self):
        for line in self.proc.stdout:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) >= 9 and parts[1].replace(".", "").isdigit():
                self.rows.append((time.monotonic(), parts))

    def __enter__(self):
        import threading
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--id={self.gpu}", f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", str(self.period)],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True, bufsize=1)
            self.thread = threading.Thread(target=self._reader, daemon=True)
            self.thread.start()
            deadline = time.monotonic() + 10.0
            while not self.rows and time.monotonic() < deadline and self.proc.poll() is None:
                time.sleep(0.01)
        except Exception:
            self.proc = None
        return self

    def mark(self, which):
        if which == "start":
            self.t0 = time.monotonic()
        else:
            self.t1 = time.monotonic()
            time.sleep(2.5 * self.period / 1000.0)  # let the row after the region arrive

    def __exit__(self, *exc):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
        if self.thread:
            self.thread.join(timeout=2)

    def summary(self):
        rows = list(self.rows)
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}
        t0 = self.t0 if self.t0 is not None else rows[0][0]
        t1 = self.t1 if self.t1 is not None else rows[-1][0]
        inside = [r for t, r in rows if t0 <= t <= t1]
        before = [r for t, r in rows if t < t0][-1:]
        after = [r for t, r in rows if t > t1][:1]
        sel = before + inside + after
        sm = [float(r[1]) for r in sel]
        smax = max(float(r[2]) for r in sel)

        def power(r):
            try:
                return float(r[3])
            except ValueError:
                return 0.0
        loaded = [s for s, r in zip(sm, sel) if power(r) > 250.0] or sm
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({n for r in sel for n, v in zip(names, r[5:9]) if v.lower() == "active"})
        return {"sm_mhz": statistics.median(loaded), "sm_max_mhz": smax, "reasons": reasons,
                "samples": len(sel), "samples_inside": len(inside),
                "timed_region_s": round(t1 - t0, 4), "period_ms": self.period}


# The JSON line is the only thing bench.py may put on stdout; NCCL's init banner ("NCCL version
# ...", printed on stdout by every communicator init, ours and torch's) and any other library
# chatter are sent to stderr by pointing fd 1 there for the run.
_JSON_OUT = None


def emit(line):
    out = _JSON_OUT if _JSON_OUT is not None else sys.stdout
    print(json.dumps(line), file=out, flush=True)


def quiet_stdout():
    global _JSON_OUT
    if _JSON_OUT is None:
        sys.stdout.flush()
        _JSON_OUT = os.fdopen(os.dup(1), "w")
        os.dup2(2, 1)


def algorithmic_mma(ndim, nk, tf, engine, points, tc_planes):
    """DMMA.8x8x4 per pass over `points` outputs: Eq 13 generalised by
    reading A7 (N fragments) and 3D planes for TC_S2R; 4x2/2x4 blocks for TC_TILE 2D/3D and
    8-output Toeplitz blocks (K = nk + 7 rounded up to 4) for TC_TILE 1D."""
    if engine == "tc_tile" and ndim == 1:
        return points / 64 * math.ceil((nk + 7) / 4)
    if engine == "tc_s2r":
        sw = nk + 1
        nf = (sw + 7) // 8
        k = nk if ndim == 1 else nk * nk
        return points / (8 * sw) * 2 * math.ceil(k / 4) * nf * tc_planes
    if engine == "tc_tile" and ndim == 3 and tf == 2:
        # 3D Tf = 2 by temporal blocking (k_tile3d_tb): two steps of the base stencil (nk = 3,
        # 4x2 blocks, 6 DMMAs per 64 outputs per TC plane); the recomputed halo is overhead
        return 2 * points / 64 * 6 * tc_planes
    if engine == "tc_tile":
        # the block shape of smaller K (planner.cpp): 2x4 for nk = 5, 9, 13; 4x2 otherwise
        kdim = lambda a, b: (a + nk - 1) * 4 * math.ceil((b + nk - 1) / 4)
        return points / 64 * (min(kdim(4, 2), kdim(2, 4)) // 4) * tc_planes
    return 0.0


def tc_planes_of(name, w):
    s = synth.SHAPES[name]
    if s.ndim != 3:
        return 1
    return sum(int(np.count_nonzero(w[z]) > 1) for z in range(w.shape[0]))


def cpu_oracle_sample(shape, ext, T, bc, w, budget_s=12.0, rows=None):
    """Time the oracle (as it stands) on the host cores: the full grid of this config (or a
    slab of it) for as many base steps as fit in ~budget_s."""
    import oracle
    cores = len(os.sched_getaffinity(0))
    u0 = synth.grid(ext, rows=rows)
    _, s1 = oracle.run(u0, w, bc, 1, nthreads=cores, return_seconds=True)
    steps = int(max(1, min(T, budget_s / max(s1, 1e-6))))
    _, secs = oracle.run(u0, w, bc, steps, nthreads=cores, return_seconds=True)
    pts = u0.size
    return {"value": steps * pts / secs / 1e9, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"{shape} {'x'.join(map(str, u0.shape))}, {bc}, {steps} of T={T} base steps "
                      f"(plain-C oracle, OpenMP {cores} threads, {secs:.1f} s)"}


def run_reference(args, cfg_name):
    """The reference arm: the oracle (as it stands) on the host cores, rank 0 only.  Each step is
    a bounded sample of the workload: the full grid for as many base steps as fit in a per-step
    budget chosen so that W + K steps end within ~2 minutes."""
    import oracle
    shape, ext, T, bc, _ = CONFIGS[cfg_name]
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    w = synth.physical_weights(shape)
    nranks = args.gpus
    if nranks > 1:
        ext = (ext[0] * nranks,) + tuple(ext[1:])
    cores = len(os.sched_getaffinity(0))
    u0 = synth.grid(ext)
    _, s1 = oracle.run(u0, w, bc, 1, nthreads=cores, return_seconds=True)
    budget = min(8.0, 120.0 / (args.warmup + args.steps))
    steps = int(max(1, min(T, budget / max(s1, 1e-6))))
    vals, secs_all = [], []
    for i in range(args.warmup + args.steps):
        _, secs = oracle.run(u0, w, bc, steps, nthreads=cores, return_seconds=True)
        if i >= args.warmup:
            vals.append(steps * u0.size / secs / 1e9)
            secs_all.append(secs)
    value = statistics.median(vals)
    sample = (f"{shape} {'x'.join(map(str, u0.shape))}, {bc}, {steps} of T={T} base steps per step "
              f"(plain-C oracle, OpenMP {cores} threads)")
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1e3 * statistics.median(secs_all) * T / steps,
            "ms_per_step_note": (f"extrapolated to the full T={T} from the {steps} base steps each timed "
                                 "step runs (the rate is measured; the full-T time is not)"
                                 if steps < T else "measured"),
            "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic (splitmix64 seed 20240302, dyadic physical weights)",
            "config": {"workload": cfg_name, "grid": list(ext), "T": T, "bc": bc,
                       "parallelism": "oracle on host cores"},
            "cpu_baseline": {"kind": "oracle", "cores": cores, "sample": sample, "value": value,
                             "unit": UNIT},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    emit(line)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="csx", choices=["csx", "reference"])
    ap.add_argument("--config", default=DEFAULT, choices=sorted(CONFIGS) + ["custom"])
    ap.add_argument("--engine", default="auto", choices=["auto", "tc_s2r", "tc_tile", "direct"])
    ap.add_argument("--shape", default=None, help="custom workload: stencil name (synth.SHAPES)")
    ap.add_argument("--grid", default=None, help="custom workload: comma-separated extents")
    ap.add_argument("--T", type=int, default=None, help="custom workload: base time steps")
    ap.add_argument("--bc", default=None, choices=["fixed", "periodic"])
    ap.add_argument("--fuse", type=int, default=None, help="override the fusion depth Tf")
    ap.add_argument("--s2r-variant", default="V", choices=["I", "II", "III", "IV", "V"],
                    help="TC_S2R breakdown variant (Fig 6): II CUDA-core tessellation, III no padding/"
                         "no dirty bits, IV padding, V full")
    ap.add_argument("--exchange", default="both", choices=["both", "peer", "nccl"],
                    help="N > 1 halo exchange: NCCL send/recv (the north_star path), SM peer stores "
                         "over NVLink, or both (default: the line's value is the NCCL run, the peer-store "
                         "run is reported beside it under 'exchange_peer')")
    ap.add_argument("--decomp", default="slab", choices=["slab", "pencil"],
                    help="multi-GPU decomposition: slabs along the slowest axis (default) or a "
                         "p0 x p1 pencil / block grid over the two slowest axes (NCCL exchange; "
                         "--gpus 1 runs the 1 x 1 pencil path)")
    ap.add_argument("--no-graph", dest="graph", action="store_false",
                    help="single GPU: launch every pass eagerly instead of replaying the step's "
                         "pass sequence as one CUDA graph (csx_plan_set_graph, the default)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-comparator", action="store_true")
    ap.add_argument("--prof-every", type=int, default=8,
                    help="time every n-th dominant-kernel launch with CUDA events (0: none)")
    args = ap.parse_args()
    quiet_stdout()
    if args.warmup < 3:
        args.warmup = 3  # timing rule: W >= 3

    if args.shape or args.grid or args.T or args.bc or args.fuse is not None:
        shape0, ext0, T0, bc0, tf0 = CONFIGS[args.config]
        shape = args.shape or shape0
        ext = tuple(int(v) for v in args.grid.split(",")) if args.grid else ext0
        if len(ext) != synth.SHAPES[shape].ndim:
            raise SystemExit("--grid must have one extent per axis of --shape")
        name = f"{shape}_{'x'.join(map(str, ext))}_T{args.T or T0}"
        CONFIGS[name] = (shape, ext, args.T or T0, args.bc or bc0, tf0 if args.fuse is None else args.fuse)
        args.config = name
    if args.impl == "reference":
        run_reference(args, args.config)
        return

    import torch
    import torch.distributed as dist
    import paper_conf_ppopp_chenlwbwmyzcy24_b200 as csx

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world}")
    # CSX_BENCH_SHARE_GPU=1: every rank on cuda:0 (exercises the N > 1 path on a 1-GPU box;
    # time-sliced, so not a scaling number)
    share = os.environ.get("CSX_BENCH_SHARE_GPU") == "1"
    device = 0 if share else local
    torch.cuda.set_device(device)
    red_dev = "cpu" if share else "cuda"  # gloo (shared-GPU test mode) reduces on CPU
    if world > 1:
        if share:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))

    shape, ext, T, bc, tf = CONFIGS[args.config]
    s = synth.SHAPES[shape]
    w = synth.physical_weights(shape)
    pencil = args.decomp == "pencil"
    if pencil:
        if s.ndim < 2:
            raise SystemExit("--decomp pencil needs a 2D or 3D shape")
        p1 = max(d for d in range(1, int(math.isqrt(world)) + 1) if world % d == 0)
        p0 = world // p1
        gext = (ext[0] * p0, ext[1] * p1) + tuple(ext[2:])  # weak scaling: ext per GPU
    else:
        gext = (ext[0] * world,) + tuple(ext[1:])  # weak scaling: ext per GPU
    plan = csx.Plan(gext, w, shape=s.kind, bc=bc, fuse_steps=tf, engine=args.engine)
    if args.s2r_variant == "I":
        plan.set_s2r_variant(padding=3, dirty_bits=True)
    elif args.s2r_variant == "II":
        plan.set_s2r_variant(padding=2, dirty_bits=True)
    elif args.s2r_variant != "V":
        plan.set_s2r_variant(padding=args.s2r_variant == "IV", dirty_bits=False)
    info = plan.info()
    engine = info["engine_name"]
    stream = torch.cuda.current_stream()
    comm = None
    exchange = None
    if pencil:
        exchange = f"nccl pencil {p0}x{p1}"
        uid = [csx.csx_nccl_unique_id() if rank == 0 else None]
        if world > 1:
            dist.broadcast_object_list(uid, src=0)
        comm = csx.csx_comm_create(uid[0], rank, world)
        lo, hi = plan.shard_box(rank, p0, p1)
        u0 = np.ascontiguousarray(synth.grid(gext, rows=(lo[0], hi[0]))[:, lo[1]:hi[1]])
    elif world > 1:
        # shared-GPU test mode (ranks on one GPU): NCCL cannot put two ranks on one device
        exchange = "peer" if (args.exchange == "peer" or share) else "nccl"
        if exchange == "peer":
            # halo exchange by SM peer stores over NVLink (CUDA IPC), epoch flags in peer memory;
            # if the IPC mapping is refused, every rank switches to the NCCL exchange
            err = None
            try:
                plan.peer_setup(rank, world)
            except Exception as e:  # noqa: BLE001  (reported in the JSON line)
                err = repr(e)
            errs = [None] * world
            dist.all_gather_object(errs, err)
            if any(errs):
                msg = next(e for e in errs if e)
                if share:  # shared-GPU test mode: NCCL cannot put two ranks on one GPU
                    raise SystemExit(f"peer setup failed: {msg}")
                print(f"[bench] peer setup failed, using NCCL: {msg}", file=sys.stderr)
                exchange = "nccl (peer setup failed: " + msg[:120] + ")"
                plan.close()
                plan = csx.Plan(gext, w, shape=s.kind, bc=bc, fuse_steps=tf, engine=args.engine)
        if not exchange.startswith("peer"):
            uid = [csx.csx_nccl_unique_id() if rank == 0 else None]
            dist.broadcast_object_list(uid, src=0)
            comm = csx.csx_comm_create(uid[0], rank, world)
        lo, hi = plan.shard_rows(rank, world)
        u0 = synth.grid(gext, rows=(lo, hi))
    if not pencil and world == 1:
        u0 = synth.grid(gext)
    d_in = torch.from_numpy(u0).cuda()
    d_out = torch.empty_like(d_in)
    n_local = u0.size

    def step():
        if pencil:
            plan.run_sharded_pencil(comm, p0, p1, d_in, d_out, T, n_local, stream)
        elif world == 1:
            plan.run(d_in, d_out, T, stream)
        elif comm is None:
            plan.run_sharded_peer(d_in, d_out, T, n_local, stream)
        else:
            plan.run_sharded(comm, d_in, d_out, T, n_local, stream)

    def barrier_sync():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    for _ in range(args.warmup):
        step()
    barrier_sync()
    # the dominant kernel's duration is sampled live: every --prof-every-th main-pass launch is
    # bracketed by CUDA events on its stream (events between kernels break PDL chaining)
    graph = args.graph and world == 1 and not pencil
    if graph:  # the pass sequence is captured by the warm-up steps and replayed in the timed ones
        plan.set_graph(True)
        for _ in range(2):
            step()
        barrier_sync()
    # (graph replay carries no per-kernel events: the dominant kernel is then timed in one extra
    # eager step after the timed region)
    csx.csx_profile_enable(plan.handle, 0 if graph else args.prof_every)
    csx.csx_profile_read(plan.handle, reset=True)
    # Timing rule: grids larger than L2 (126 MB) need no flush; smaller ones get a 256 MB write
    # between timed steps, outside the per-step CUDA-event windows.
    flush = None
    if 2 * u0.nbytes < 256 << 20:
        flush = torch.empty(32 << 20, dtype=torch.float64, device="cuda")
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
           for _ in range(args.steps)]
    with ClockSampler(device) as clk:
        barrier_sync()
        clk.mark("start")
        for e0, e1 in evs:
            if flush is not None:
                flush.fill_(1.0)
            e0.record(stream)
            step()
            e1.record(stream)
        barrier_sync()
        clk.mark("end")
    ms_total = sum(e0.elapsed_time(e1) for e0, e1 in evs)
    tc_ms, tc_launches, launches = csx.csx_profile_read(plan.handle, reset=True)
    eager_ms = None  # graph mode: duration of the extra eager (profiled) step
    if graph and args.prof_every > 0:
        csx.csx_profile_enable(plan.handle, args.prof_every)
        ee0 = torch.cuda.Event(enable_timing=True)
        ee1 = torch.cuda.Event(enable_timing=True)
        if flush is not None:
            flush.fill_(1.0)
        ee0.record(stream)
        step()
        ee1.record(stream)
        torch.cuda.synchronize()
        eager_ms = ee0.elapsed_time(ee1)
        tc_ms, tc_launches, _ = csx.csx_profile_read(plan.handle, reset=True)
        plan.set_graph(False)
    csx.csx_profile_enable(plan.handle, False)
    if world > 1:
        t = torch.tensor([ms_total], device=red_dev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms_total = float(t.item())
    ms_step = ms_total / args.steps
    points = int(np.prod(gext))
    value = T * points / (ms_step * 1e-3) / 1e9

    # ---- roofline of the dominant kernel (the main-pass TC kernel) ----
    hbm, hbm_src, dmma, dmma_src = peaks()
    nk, tfm = info["nk"], info["fuse_steps"]
    local_points = n_local
    tcp = tc_planes_of(shape, w)
    roof = None
    if tc_launches > 0 and engine in ("tc_s2r", "tc_tile"):
        avg_s = tc_ms / tc_launches * 1e-3
        if eager_ms:
            # graph replay carries no per-kernel events: the dominant kernel's share of the extra
            # eager step, applied to the replayed step's time (an eager step is slower than its
            # replay when it is launch-bound, e.g. the 1D configs' short passes)
            kshare = min(1.0, tc_ms / eager_ms)
            avg_eager_ms = tc_ms / tc_launches
            avg_s = kshare * ms_step / tc_launches * 1e-3
        mma = algorithmic_mma(s.ndim, nk, tfm, engine, local_points, tcp)
        mma_src = ("Eq 13 generalised (reading A7, 3D planes)" if engine == "tc_s2r" else
                   "TC_TILE block count: K of the a x b output block / 4 per 64 outputs")
        flops = 512.0 * mma
        byts = 16.0 * local_points
        tc_bound = (flops / (dmma * 1e12)) >= (byts / (hbm * 1e9))
        traffic = None
        tr = load_json(os.path.join(ROOT, "profiles", "traffic.json")) or {}
        key = f"{args.config}:{engine}"
        if key in tr:
            traffic = tr[key]
        # the launch-list name of the dominant kernel (k_tile2d / k_s2r3d / k_direct1d ...)
        kname = f"k_{ {'tc_tile': 'tile', 'tc_s2r': 's2r'}.get(engine, engine)}{s.ndim}d<nk={nk}>"
        if tc_bound:
            achieved = flops / avg_s / 1e12
            roof = {"bound": "tensor", "achieved": achieved, "peak": dmma, "unit": "TFLOP/s",
                    "frac": achieved / dmma, "traffic": traffic, "peak_source": dmma_src,
                    "kernel": kname, "avg_launch_ms": avg_s * 1e3,
                    "launches": tc_launches,
                    "per_launch": f"{mma:.0f} DMMA.8x8x4 x 512 flop ({mma_src})",
                    "hbm_frac": byts / avg_s / 1e9 / hbm}
        else:
            achieved = byts / avg_s / 1e9
            roof = {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s",
                    "frac": achieved / hbm, "traffic": traffic, "peak_source": hbm_src,
                    "kernel": kname, "avg_launch_ms": avg_s * 1e3,
                    "launches": tc_launches,
                    "per_launch": f"16 B x {local_points} points (1 read + 1 write per pass)",
                    "tensor_frac": flops / avg_s / 1e12 / dmma}
        if eager_ms:
            roof["tc_share_of_step"] = kshare
            roof["timing"] = ("dominant-kernel share of one eager profiled step x the replayed "
                              "step time / launches per step")
            roof["avg_launch_ms_eager"] = avg_eager_ms
            roof["eager_step_ms"] = eager_ms
        else:
            roof["tc_share_of_step"] = tc_ms / ms_total if ms_total > 0 else None
            roof["timing"] = "CUDA events around sampled launches inside the timed steps"
        roof["timed_every"] = args.prof_every
        # hardware counters of the same kernel from the committed ncu pass (scripts/dmma_counters.py:
        # one main-pass launch of this config and engine): DMMA instructions executed vs the count
        # the planner states, DMMA-pipe active %, DRAM bytes vs algorithmic
        hw = (load_json(os.path.join(ROOT, "profiles", "dmma_counters.json")) or {}).get(key)
        if hw:
            roof["ncu"] = {
                "kernel": hw.get("kernel"),
                "dmma_inst_per_launch": hw.get("sm__inst_executed_pipe_tensor_subpipe_dmma.sum"),
                "dmma_inst_planner": (hw.get("info") or {}).get("mma_per_pass"),
                "dmma_inst_vs_planner": hw.get("dmma_inst_vs_planner"),
                "dmma_pipe_active_pct": hw.get(
                    "sm__pipe_tensor_subpipe_dmma_cycles_active.avg.pct_of_peak_sustained_elapsed"),
                "fp64_shared_pipe_active_pct": hw.get(
                    "sm__pipe_shared_cycles_active.avg.pct_of_peak_sustained_elapsed"),
                "dram_bytes_per_launch": hw.get("dram_bytes"),
                "dram_vs_algorithmic": hw.get("dram_vs_algorithmic"),
                "source": "profiles/dmma_counters.json (ncu --metrics, one main-pass launch, cold L2)"}

    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic (splitmix64 seed 20240302, dyadic physical weights)",
            "config": {"workload": args.config, "shape": shape, "grid": list(gext), "T": T, "bc": bc,
                       "fuse_steps": tfm, "nk": nk, "engine": engine, "cuda_graph": graph,
                       "s2r_variant": args.s2r_variant if engine == "tc_s2r" else None,
                       "parallelism": (f"pencil{p0}x{p1}" if pencil else f"slab{world}" if world > 1 else "single"),
                       "exchange": exchange,
                       "l2": ("L2 flushed (256 MB write) between timed steps" if flush is not None
                              else f"inputs larger than L2 ({u0.nbytes >> 20} MB per grid vs 126 MB); no flush")},
            "gpu_launches": int(launches), "roofline": roof}

    # ---- rank-0 extras: clocks, comparator, e2e, cpu baseline ----
    clocks = clk.summary()
    line["clocks"] = clocks
    if rank == 0 and world == 1 and not args.no_comparator and engine != "direct":
        try:
            # same protocol as the TC line: warm-up runs, then K timed steps with the same L2
            # flush between them (small grids) and the same CUDA-graph replay
            # the comparator at ITS OWN best fusion depth (csx_auto_fuse_steps for DIRECT)
            cplan = csx.Plan(gext, w, shape=s.kind, bc=bc, engine="direct")
            ctf = cplan.info()["fuse_steps"]
            if graph:
                cplan.set_graph(True)
            for _ in range(args.warmup):
                cplan.run(d_in, d_out, T, stream)
            torch.cuda.synchronize()
            cev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                   for _ in range(args.steps)]
            for e0, e1 in cev:
                if flush is not None:
                    flush.fill_(1.0)
                e0.record(stream)
                cplan.run(d_in, d_out, T, stream)
                e1.record(stream)
            torch.cuda.synchronize()
            cms = sum(e0.elapsed_time(e1) for e0, e1 in cev) / args.steps
            cplan.close()
            useful = 2.0 * s.points
            cval = T * points / (cms * 1e-3) / 1e9
            fp = load_json(os.path.join(ROOT, "PEAKS_FP64.json")) or {}
            dfma = fp.get("dfma_tflops_sustained") or fp.get("dfma_tflops") or 37.0
            hbm_roof = hbm * ctf / 16.0             # GSt/s: 16 B per point per pass of Tf steps
            dfma_roof = dfma * 1e3 / useful          # GSt/s: useful DFMA flops only (no recompute)
            line["comparator"] = {"engine": "direct (CUDA-core DFMA, temporal blocking)",
                                  "value": cval, "unit": UNIT, "ms_per_step": cms,
                                  "useful_flops_per_point_step": useful, "fuse_steps": ctf,
                                  "roof_gsts": min(hbm_roof, dfma_roof),
                                  "roof": "hbm" if hbm_roof < dfma_roof else "dfma",
                                  "frac": cval / min(hbm_roof, dfma_roof),
                                  "hbm_roof_gsts": hbm_roof, "dfma_roof_gsts": dfma_roof,
                                  "dfma_peak_tflops": dfma}
        except Exception as e:  # report, do not hide
            line["comparator"] = {"error": str(e)}
    if not args.no_e2e:
        # end to end through the public host-buffer API: pinned host in, H2D, run, D2H
        if world == 1:
            h_in = torch.from_numpy(u0).pin_memory().numpy()
            h_out = torch.empty(u0.shape, dtype=torch.float64).pin_memory().numpy()
            plan.run_host(h_in, T, h_out, stream)
            e_steps = max(1, min(args.steps, 3))
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            e0.record(stream)
            for _ in range(e_steps):
                plan.run_host(h_in, T, h_out, stream)
            e1.record(stream)
            torch.cuda.synchronize()
            ems = e0.elapsed_time(e1) / e_steps
            h_chunks, h2d_b, d2h_b = plan.host_last()
            if h_chunks > 1:  # the C-ABI's ghost-zone chunk pipeline (include/csx.h csx_run_host)
                dev = d_out.cpu().numpy()  # the device run's result (same input and T)
                if np.max(np.abs(h_out - dev)) > 1e-12 * np.max(np.abs(dev)):
                    raise SystemExit("chunked csx_run_host result differs from the device run")
                how = (f"{h_chunks} ghost-zone chunks along the slowest axis, H2D(k+1) / run(k) / "
                       "D2H(k-1) overlapped on three streams")
            else:
                how = "H2D + run + D2H serialised on one stream"
            sync_line = {"value": T * points / (ems * 1e-3) / 1e9, "unit": UNIT, "ms_per_step": ems,
                         "api": f"csx_run_host through the C-ABI (pinned host buffers; {how}; timed by "
                                "CUDA events around the calls)", "chunks": h_chunks}
            # A stream of grids through the same public calls: every step copies its own input
            # host->device and its whole result device->host, but step i+1's H2D and step i-1's
            # D2H (PCIe is full duplex) run on their own streams while step i computes.
            plan.set_graph(False)  # alternating buffers would re-capture every step
            K = max(args.steps, 12)
            s_in, s_out = torch.cuda.Stream(), torch.cuda.Stream()
            hin = [torch.from_numpy(u0).pin_memory() for _ in range(2)]
            hout = [torch.empty(u0.shape, dtype=torch.float64).pin_memory() for _ in range(2)]
            din = [d_in, torch.empty_like(d_in)]
            dout = [d_out, torch.empty_like(d_out)]
            ev_in = [torch.cuda.Event() for _ in range(2)]
            ev_run = [torch.cuda.Event() for _ in range(2)]
            ev_out = [torch.cuda.Event() for _ in range(2)]
            plan.run(d_in, d_out, T, stream)
            ref = d_out.clone()  # this config's result for the check below (same input and T)
            torch.cuda.synchronize()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(s_in)
            for i in range(K):
                b = i % 2
                if i >= 2:
                    s_in.wait_event(ev_run[b])    # din[b] was read by step i-2
                with torch.cuda.stream(s_in):
                    din[b].copy_(hin[b], non_blocking=True)
                ev_in[b].record(s_in)
                stream.wait_event(ev_in[b])
                if i >= 2:
                    stream.wait_event(ev_out[b])  # dout[b] was read by step i-2's D2H
                plan.run(din[b], dout[b], T, stream)
                ev_run[b].record(stream)
                s_out.wait_event(ev_run[b])
                with torch.cuda.stream(s_out):
                    hout[b].copy_(dout[b], non_blocking=True)
                ev_out[b].record(s_out)
            e1.record(s_out)
            torch.cuda.synchronize()
            pms = e0.elapsed_time(e1) / K
            if not torch.equal(hout[(K - 1) % 2], ref.cpu()):
                raise SystemExit("pipelined e2e result differs from the device run")
            sync_line.update({"h2d_bytes_per_step": int(h2d_b), "d2h_bytes_per_step": int(d2h_b),
                              "steps": e_steps})
            sync_line["pipelined"] = {
                "value": T * points / (pms * 1e-3) / 1e9, "unit": UNIT, "ms_per_step": pms,
                "api": "Plan.run (csx_run) + torch pinned copies, pipelined over "
                       f"{K} steps: H2D(i+1) and D2H(i-1) overlap run(i)"}
            line["e2e"] = sync_line
        else:
            h_in = torch.from_numpy(u0).pin_memory()
            h_out = torch.empty(u0.shape, dtype=torch.float64).pin_memory()
            barrier_sync()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            d_in.copy_(h_in, non_blocking=True)
            step()
            h_out.copy_(d_out, non_blocking=True)
            e1.record(stream)
            barrier_sync()
            ems = torch.tensor([e0.elapsed_time(e1)], device=red_dev, dtype=torch.float64)
            dist.all_reduce(ems, op=dist.ReduceOp.MAX)
            ems = float(ems.item())
            line["e2e"] = {"value": T * points / (ems * 1e-3) / 1e9, "unit": UNIT,
                           "h2d_bytes_per_step": int(u0.nbytes), "d2h_bytes_per_step": int(u0.nbytes),
                           "api": "torch pinned copies + csx_run_sharded" + ("_peer" if comm is None else ""),
                           "ms_per_step": ems}
    if world > 1 and not pencil and args.exchange == "both" and not share:
        # the same weak-scaled step with the halo exchange fused into SM peer stores over NVLink
        # (csx_run_sharded_peer), timed the same way (max over ranks); the line's value is the
        # NCCL run above (the north_star path)
        peer_line = {"exchange": "peer (SM stores into the neighbours' ghost rows over NVLink, epoch flags)"}
        pplan = csx.Plan(gext, w, shape=s.kind, bc=bc, fuse_steps=tf, engine=args.engine)
        err = None
        try:
            pplan.peer_setup(rank, world)
        except Exception as e:  # noqa: BLE001  (reported in the JSON line)
            err = repr(e)
        errs = [None] * world
        dist.all_gather_object(errs, err)
        if any(errs):
            peer_line["error"] = next(e for e in errs if e)[:200]
        else:
            def pstep():
                pplan.run_sharded_peer(d_in, d_out, T, n_local, stream)
            for _ in range(args.warmup):
                pstep()
            pev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                   for _ in range(args.steps)]
            barrier_sync()
            for e0, e1 in pev:
                e0.record(stream)
                pstep()
                e1.record(stream)
            barrier_sync()
            t = torch.tensor([sum(a.elapsed_time(b) for a, b in pev)], device=red_dev, dtype=torch.float64)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            pms = float(t.item()) / args.steps
            peer_line.update({"value": T * points / (pms * 1e-3) / 1e9, "unit": UNIT, "ms_per_step": pms})
        barrier_sync()  # a neighbour's last push writes into this rank's flags: sync before freeing
        pplan.close()
        line["exchange_peer"] = peer_line
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_oracle_sample(shape, gext, T, bc, w)
    if rank == 0:
        emit(line)
    if comm is not None:
        csx.csx_comm_destroy(comm)
    plan.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
