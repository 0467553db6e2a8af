"""Regenerate the measured tables of profiles/r02/README.md from the files the round-2 GPU pass
(scripts/r02_full2.sh) brought back: bench lines, ncu DMMA / DRAM counters, ncu --set full
briefs, the launch list.  The hand-written notes at the end (from '## Notes') are kept.
usage: python scripts/profiles_readme_r02.py"""
import glob
import json
import os
import re
import subprocess
import sys

D = os.path.join("profiles", "r02")
readme = os.path.join(D, "README.md")
old = open(readme).read() if os.path.exists(readme) else ""
notes = old[old.index("## Notes"):] if "## Notes" in old else "## Notes\n"


def lines(path):
    out = []
    if not os.path.exists(path):
        return out
    for ln in open(path):
        try:
            out.append(json.loads(ln))
        except ValueError:
            pass
    return out


def bench_table(rows):
    t = ["| workload | engine | Tf | nk | GSt/s | bound | frac | DMMA % (ncu) | DRAM / alg. | comparator (Tf) | comp. frac | e2e csx_run_host | e2e pipelined | SM MHz |",
         "|---|---|---|---|---|---|---|---|---|---|---|---|---|---|"]
    for d in rows:
        if "error" in d:
            t.append(f"| {d.get('config')} | error | | | | | | | | | | | | |")
            continue
        c = d["config"]
        r = d.get("roofline") or {}
        n = r.get("ncu") or {}
        cm = d.get("comparator") or {}
        e = d.get("e2e") or {}
        dv = n.get("dram_vs_algorithmic")
        t.append(f"| {c['workload']} | {c['engine']} | {c['fuse_steps']} | {c['nk']} | {d['value']:.1f} | "
                 f"{r.get('bound', '-')} | {r.get('frac', 0):.3f} | {n.get('dmma_pipe_active_pct', '-')} | "
                 f"{'' if dv is None else f'{dv:.3f}'} | "
                 f"{'' if not cm.get('value') else f'{cm['value']:.1f} ({cm.get('fuse_steps')})'} | "
                 f"{'' if not cm.get('frac') else f'{cm['frac']:.2f}'} | "
                 f"{'' if not e.get('value') else f'{e['value']:.1f}'} | "
                 f"{'' if not (e.get('pipelined') or {}).get('value') else f'{e['pipelined']['value']:.1f}'} | "
                 f"{d['clocks'].get('sm_mhz')} {','.join(d['clocks'].get('reasons') or [])} |")
    return "\n".join(t)


def dmma_table(path):
    if not os.path.exists(path):
        return ""
    dm = json.load(open(path))
    t = ["| config:engine | kernel | DMMA inst / launch | planner | ratio | DMMA pipe % | FP64 shared pipe % | DRAM MB | DRAM / alg. | us (cold) |",
         "|---|---|---|---|---|---|---|---|---|---|"]
    for k in sorted(dm):
        v = dm[k]
        kn = (v.get("kernel") or "")[:60]
        inf = v.get("info") or {}
        us = v.get("gpu__time_duration.sum")
        unit = v.get("gpu__time_duration.sum:unit", "ns")
        us = us / 1e3 if unit == "ns" else (us * 1e3 if unit == "ms" else us)
        t.append(f"| {k} | `{kn}` | {v.get('sm__inst_executed_pipe_tensor_subpipe_dmma.sum')} | "
                 f"{inf.get('mma_per_pass')} | {v.get('dmma_inst_vs_planner')} | "
                 f"{v.get('sm__pipe_tensor_subpipe_dmma_cycles_active.avg.pct_of_peak_sustained_elapsed')} | "
                 f"{v.get('sm__pipe_shared_cycles_active.avg.pct_of_peak_sustained_elapsed')} | "
                 f"{(v.get('dram_bytes') or 0) / 1e6:.1f} | {v.get('dram_vs_algorithmic') or 0:.3f} | "
                 f"{us:.1f} |")
    return "\n".join(t)


def brief_table():
    t = ["| capture | kernel | us (cold) | DRAM rd GB | DRAM wr GB | DMMA % active | regs | smem ld conflicts | L2 hit % | top stalls |",
         "|---|---|---|---|---|---|---|---|---|---|"]
    for f in sorted(glob.glob(os.path.join(D, "brief", "brief_*.txt"))):
        s = open(f).read()

        def num(k):
            m = re.search(re.escape(k) + r"\s+([0-9.]+)", s)
            return float(m.group(1)) if m else float("nan")
        kn = s.splitlines()[0][:50] if s else ""
        us = num("gpu__time_duration.sum")
        rd, wr = num("dram__bytes_read.sum"), num("dram__bytes_write.sum")
        if rd > 50:
            rd, wr = rd / 1000, wr / 1000
        st = (re.search(r"stalls: (.*)", s) or [None, ""])[1]
        t.append(f"| {os.path.basename(f)[6:-4]} | `{kn}` | {us:.1f} | {rd:.3f} | {wr:.3f} | "
                 f"{num('sm__pipe_tensor_subpipe_dmma_cycles_active.avg.pct_of_peak_sustained_active'):.1f} | "
                 f"{num('launch__registers_per_thread'):.0f} | "
                 f"{num('l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum'):.0f} | "
                 f"{num('lts__t_sector_hit_rate.pct'):.1f} | {st} |")
    return "\n".join(t)


launch = ""
lc = os.path.join(D, "launches_box2d9p.csv")
if os.path.exists(lc):
    launch = subprocess.run([sys.executable, "scripts/launch_summary.py", lc], capture_output=True, text=True).stdout

out = f"""# Round 2 profiles (B200, sm_100a)

Measured at HEAD through gpurun (`scripts/r02_final2.sh`; earlier passes `r02_full2.sh`, `r02_final.sh`): the whole GPU suite (`gpu_all.log`),
`smoke()` (`smoke.log`), one bench line per config (`bench_all.jsonl`: TC_TILE / auto engine with
the CUDA-core comparator at its own fusion depth, e2e through `csx_run_host`, the ncu counters
of the committed DMMA pass), the paper's layout (`bench_s2r.jsonl`), the plain `python bench.py`
line (`bench_default.json`), the reference arm (`bench_reference.json`: the oracle on the
host cores), the DMMA / FP64-pipe / DRAM counters of every dominant kernel
(`dmma_counters.json`, `scripts/dmma_counters.py`), `ncu --set full` briefs of the round-2
kernels with their SASS stall maps (`brief/`), sanitizers of earlier passes (`*check*.txt`) and the launch list of the default bench.  ncu
runs are cold-cache and serialised: compare shares and counters, not absolute times.
This file's tables are regenerated by `scripts/profiles_readme_r02.py`.

## Bench, every config (`bench_all.jsonl`)

{bench_table(lines(os.path.join(D, 'bench_all.jsonl')))}

## The paper's layout, TC_S2R (`bench_s2r.jsonl`)

{bench_table(lines(os.path.join(D, 'bench_s2r.jsonl')))}

## Other lines (`bench_extra.jsonl`)

{bench_table(lines(os.path.join(D, 'bench_extra.jsonl')))}

## DMMA instructions and pipe activity per dominant kernel (`dmma_counters.json`)

{dmma_table(os.path.join(D, 'dmma_counters.json'))}

## ncu --set full briefs (`brief/`)

{brief_table()}

## Launch list of the default bench (Box-2D9P 10240², T = 100)

```
{launch.strip()}
```

{notes}"""
open(readme, "w").write(out)
print("wrote", readme)
