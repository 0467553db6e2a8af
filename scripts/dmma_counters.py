"""DMMA / FP64-pipe / DRAM hardware counters of the dominant kernel of each (config, engine),
against the planner's DMMA count (SURVEY §8(d) "DMMA pipe active %"; Eq 13, PAPER.md
P.1512-1524).  Runs on the GPU box:

  python scripts/dmma_counters.py --out gpurun_out/r02b/dmma.json  [config:engine ...]

For each case: `ncu --metrics <below> -k regex:<kernel> -s <skip> -c 1` around scripts/one_run.py
(one eager csx_run; skip lands on a main pass), the launch's counters, and the plan's
info["mma_per_pass"] (the DMMAs the planner says that pass executes).
"""
import argparse
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
NCU = "/usr/local/cuda/bin/ncu"
METRICS = [
    "gpu__time_duration.sum",
    "sm__inst_executed_pipe_tensor_subpipe_dmma.sum",
    "sm__pipe_tensor_subpipe_dmma_cycles_active.avg.pct_of_peak_sustained_elapsed",
    "sm__pipe_shared_cycles_active.avg.pct_of_peak_sustained_elapsed",
    "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_elapsed",
    "sm__inst_executed_pipe_fp64.sum",
    "dram__bytes_read.sum",
    "dram__bytes_write.sum",
    "sm__cycles_elapsed.avg.per_second",
]
DEFAULT = [
    "box2d9p_10240:tc_tile", "box2d9p_10240:tc_s2r", "box2d9p_10240:direct",
    "star2d13p_10240:tc_tile", "box2d49p_10240:tc_tile", "box2d49p_10240:tc_s2r",
    "box2d49p_10240_tf2:tc_tile", "heat2d_10240:tc_tile", "star2d9p_10240:tc_tile",
    "box2d25p_10240:tc_tile", "heat3d_512:tc_tile", "box3d27p_512:tc_tile", "box3d27p_512:tc_s2r",
    "box3d125p_512:tc_tile", "star3d13p_512:tc_tile", "box3d343p_512:tc_tile",
    "star3d19p_512:tc_tile", "heat1d_10240000:tc_tile", "heat1d_10240000:tc_s2r",
    "1d5p_10240000:tc_tile", "heat1d_102400000:tc_tile",
]
KRE = {("tc_tile", 1): "k_tile1d", ("tc_tile", 2): "k_tile2d", ("tc_tile", 3): "k_tile3d",
       ("tc_s2r", 1): "k_s2r1d", ("tc_s2r", 2): "k_s2r2d", ("tc_s2r", 3): "k_s2r3d",
       ("direct", 1): "k_direct1d", ("direct", 2): "k_direct2d", ("direct", 3): "k_direct3d"}


def num(v):
    try:
        return float(v.replace(",", ""))
    except ValueError:
        return None


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", required=True)
    ap.add_argument("cases", nargs="*")
    args = ap.parse_args()
    sys.path.insert(0, ROOT)
    import bench
    import synth
    res = {}
    if os.path.exists(args.out):
        res = json.load(open(args.out))
    for case in args.cases or DEFAULT:
        cfg, eng = case.split(":")
        shape = bench.CONFIGS[cfg][0]
        nd = synth.SHAPES[shape].ndim
        kre = KRE[(eng, nd)]
        log = os.path.join(os.path.dirname(args.out), f"ncu_{cfg}_{eng}.csv")
        # skip 2 launches of the kernel: the main passes follow a possible dense-source first pass
        T = 12 if nd != 1 else 60
        cmd = [NCU, "--metrics", ",".join(METRICS), "--clock-control", "none", "-k", f"regex:{kre}",
               "-s", "2", "-c", "1", "--csv", "--log-file", log,
               sys.executable, os.path.join(ROOT, "scripts", "one_run.py"), "--config", cfg,
               "--engine", eng, "--T", str(T)]
        out = subprocess.run(cmd, capture_output=True, text=True, timeout=900)
        info = None
        for line in out.stdout.splitlines():
            if line.startswith("{"):
                info = json.loads(line)
        rows = []
        if os.path.exists(log):
            txt = open(log).read()
            txt = txt[txt.find('"ID"'):] if '"ID"' in txt else ""
            rows = list(csv.DictReader(io.StringIO(txt)))
        m = {r["Metric Name"]: (num(r["Metric Value"]), r["Metric Unit"]) for r in rows}
        kname = rows[0]["Kernel Name"] if rows else None
        entry = {"kernel": kname, "info": info, "rc": out.returncode}
        for k, (v, u) in m.items():
            entry[k] = v
            entry[k + ":unit"] = u
        dm = m.get("sm__inst_executed_pipe_tensor_subpipe_dmma.sum", (None, ""))[0]
        if info and dm is not None and info.get("mma_per_pass"):
            entry["dmma_inst_vs_planner"] = dm / info["mma_per_pass"]
        if m.get("dram__bytes_read.sum") and m.get("dram__bytes_write.sum"):
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
            rb = m["dram__bytes_read.sum"][0] * scale.get(m["dram__bytes_read.sum"][1], 1)
            wb = m["dram__bytes_write.sum"][0] * scale.get(m["dram__bytes_write.sum"][1], 1)
            entry["dram_bytes"] = rb + wb
            if info:
                entry["dram_vs_algorithmic"] = (rb + wb) / (16.0 * info["points"])
        if rows == [] or out.returncode != 0:
            entry["stderr"] = out.stderr[-1500:]
        res[case] = entry
        json.dump(res, open(args.out, "w"), indent=1, sort_keys=True)
        print(case, kname, dm, info and info.get("mma_per_pass"), entry.get("dmma_inst_vs_planner"),
              m.get("sm__pipe_tensor_subpipe_dmma_cycles_active.avg.pct_of_peak_sustained_elapsed"),
              flush=True)


if __name__ == "__main__":
    main()
