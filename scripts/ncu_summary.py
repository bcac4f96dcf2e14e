"""Summarise ncu output for profiles/ (run here, on the files gpurun brought back).

    python scripts/ncu_summary.py --launches gpurun_out/launches_c2.csv \
        --rep gpurun_out/prof_c2_top.ncu-rep --out profiles/r01_c2 [--impl TRI_CHAIN]

Writes <out>_launches.md (per-kernel launch count / mean / share of the
serialised launch list), <out>_ncu.md (speed of light, memory, stall
breakdown of the captured kernel) and merges the captured kernel's DRAM bytes
per launch into profiles/ncu_summary.json (the `traffic` of bench.py's
roofline object).
"""
from __future__ import annotations

import argparse
import csv
import io
import json
import os
import subprocess
from collections import OrderedDict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def short(name: str) -> str:
    s = name.replace("sptrsv::", "").replace("k::", "")
    return s.split("(")[0].replace("void ", "")


def launches(path: str) -> tuple[str, list]:
    rows = [r for r in csv.reader(open(path)) if len(r) > 10]
    hdr, data = rows[0], rows[1:]
    ik, iv = hdr.index("Kernel Name"), hdr.index("Metric Value")
    agg: "OrderedDict[str, list]" = OrderedDict()
    for r in data:
        agg.setdefault(short(r[ik]), []).append(float(r[iv].replace(",", "")))
    ours = {k: v for k, v in agg.items() if not k.startswith("at::")}
    tot = sum(sum(v) for v in ours.values())
    lines = ["| kernel | launches | mean us | share of our kernels' time |", "|---|---|---|---|"]
    for k, v in agg.items():
        share = f"{100 * sum(v) / tot:.1f}%" if k in ours else "(L2 flush, not ours)"
        lines.append(f"| `{k}` | {len(v)} | {sum(v) / len(v) / 1e3:.2f} | {share} |")
    return "\n".join(lines), [(k, len(v), sum(v) / len(v)) for k, v in agg.items()]


def raw_metrics(rep: str) -> list[dict]:
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for vals in rows[2:]:
        res.append({h: (u, v) for h, u, v in zip(hdr, units, vals)})
    return res


def num(d, key):
    u, v = d.get(key, ("", "nan"))
    try:
        x = float(v.replace(",", ""))
    except ValueError:
        return float("nan"), u
    return x, u


def to_bytes(x, u):
    return x * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)


def summarise_rep(rep: str) -> tuple[str, list]:
    lines, recs = [], []
    for d in raw_metrics(rep):
        name = short(d.get("Kernel Name", ("", "?"))[1])
        dur, du = num(d, "gpu__time_duration.sum")
        rd = to_bytes(*num(d, "dram__bytes_read.sum"))
        wr = to_bytes(*num(d, "dram__bytes_write.sum"))
        lines.append(f"### `{name}` (grid {d.get('launch__grid_size', ('', '?'))[1]}, "
                     f"block {d.get('launch__block_size', ('', '?'))[1]})")
        lines.append("")
        lines.append("| metric | value |")
        lines.append("|---|---|")
        lines.append(f"| duration | {dur:.2f} {du} |")
        lines.append(f"| dram bytes read + write | {rd:.0f} + {wr:.0f} = {rd + wr:.0f} |")
        for key in ["sm__throughput.avg.pct_of_peak_sustained_elapsed",
                    "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
                    "dram__throughput.avg.pct_of_peak_sustained_elapsed",
                    "l1tex__throughput.avg.pct_of_peak_sustained_active",
                    "lts__t_sector_hit_rate.pct",
                    "smsp__issue_active.avg.pct_of_peak_sustained_active",
                    "sm__inst_executed.sum",
                    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
                    "smsp__sass_average_data_bytes_per_sector_mem_global_op_ld.pct",
                    "launch__registers_per_thread", "sm__warps_active.avg.pct_of_peak_sustained_active"]:
            if key in d:
                x, u = num(d, key)
                lines.append(f"| `{key}` | {x:g} {u} |")
        stalls = []
        for k in d:
            if k.startswith("smsp__average_warps_issue_stalled") and k.endswith("per_issue_active.ratio"):
                x, _ = num(d, k)
                if x == x:
                    stalls.append((x, k.replace("smsp__average_warps_issue_stalled_", "").replace(
                        "_per_issue_active.ratio", "")))
        stalls.sort(reverse=True)
        lines.append("")
        lines.append("Warp stalls (cycles per issued instruction): " +
                     ", ".join(f"{k} {x:.2f}" for x, k in stalls[:8]))
        lines.append("")
        recs.append({"kernel": name, "duration_us": dur if du == "us" else dur / 1e3 if du == "ns" else dur,
                     "dram_bytes": rd + wr})
    return "\n".join(lines), recs


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--launches")
    ap.add_argument("--rep")
    ap.add_argument("--out", required=True)
    ap.add_argument("--impl", default=None, help="bench impl name the captured kernel implements")
    ap.add_argument("--title", default="")
    ap.add_argument("--json", default=os.path.join(ROOT, "profiles", "ncu_summary.json"),
                    help="summary json the captured kernel's DRAM bytes are merged into")
    a = ap.parse_args()
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    if a.launches:
        tab, _ = launches(a.launches)
        with open(a.out + "_launches.md", "w") as f:
            f.write(f"# ncu launch list {a.title}\n\n`ncu --metrics gpu__time_duration.sum --clock-control none`"
                    f" (cold-cache, serialised; shares matter, not absolutes). Source: `{os.path.basename(a.launches)}`\n\n")
            f.write(tab + "\n")
    if a.rep:
        txt, recs = summarise_rep(a.rep)
        with open(a.out + "_ncu.md", "w") as f:
            f.write(f"# ncu --set full {a.title}\n\nSource: `{os.path.basename(a.rep)}` "
                    f"(`--set full --clock-control none --import-source on`).\n\n")
            f.write(txt + "\n")
        if a.impl and recs:
            p = a.json
            d = json.load(open(p)) if os.path.exists(p) else {}
            d.setdefault("dram_bytes_per_launch", {})[a.impl] = recs[0]["dram_bytes"]
            d.setdefault("source", {})[a.impl] = os.path.basename(a.out) + "_ncu.md"
            json.dump(d, open(p, "w"), indent=1, sort_keys=True)


if __name__ == "__main__":
    main()
