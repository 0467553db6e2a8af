"""Summarise an `ncu --set full` capture (.ncu-rep) into the numbers DESIGN.md / bench.py cite.

usage: python scripts/ncu_summary.py <report.ncu-rep> [--key config:engine --traffic profiles/traffic.json]
Prints a markdown block; with --traffic, records dram read+write bytes per launch under --key.
"""
import argparse
import collections
import csv
import io
import json
import os
import subprocess

METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("sm__cycles_elapsed.avg", "elapsed cycles"),
    ("sm__cycles_active.avg", "SM active cycles"),
    ("smsp__pipe_tensor_subpipe_dmma_cycles_active.avg", "DMMA subpipe active cycles (per SMSP)"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput % of peak"),
    ("l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum", "smem load bank conflicts"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum", "smem load wavefronts"),
    ("smsp__inst_executed.sum", "warp instructions executed"),
    ("launch__registers_per_thread", "registers / thread"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    return {h: (v, u) for h, u, v in zip(hdr, units, vals)}, rows[2][hdr.index("Kernel Name")] if "Kernel Name" in hdr else "?"


def stalls(d):
    res = []
    for k, (v, _) in d.items():
        if k.startswith("smsp__average_warps_issue_stalled_") and k.endswith("_per_issue_active.ratio"):
            try:
                res.append((float(v), k[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]))
            except ValueError:
                pass
    return sorted(res, reverse=True)[:6]


def to_bytes(v, u):
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
    return float(v.replace(",", "")) * scale


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("rep")
    ap.add_argument("--key")
    ap.add_argument("--traffic")
    args = ap.parse_args()
    d, kname = raw(args.rep)
    print(f"### {os.path.basename(args.rep)}\n\nkernel: `{kname}`\n")
    print("| metric | value |\n|---|---|")
    for m, label in METRICS:
        if m in d:
            v, u = d[m]
            print(f"| {label} (`{m}`) | {v} {u} |")
    st = stalls(d)
    print("\ntop stall reasons (warps per issue): " + ", ".join(f"{n} {v:.2f}" for v, n in st))
    if "dram__bytes_read.sum" in d and "dram__bytes_write.sum" in d:
        tb = to_bytes(*d["dram__bytes_read.sum"]) + to_bytes(*d["dram__bytes_write.sum"])
        print(f"\nDRAM traffic per launch: {tb / 1e6:.1f} MB")
        if args.traffic and args.key:
            t = {}
            if os.path.exists(args.traffic):
                t = json.load(open(args.traffic))
            t[args.key] = tb
            json.dump(t, open(args.traffic, "w"), indent=1, sort_keys=True)


if __name__ == "__main__":
    main()
