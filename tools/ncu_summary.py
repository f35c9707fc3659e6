#!/usr/bin/env python3
"""Summarise ncu captures into profiles/ (committed evidence).

  python tools/ncu_summary.py --full gpurun_out/full_r1.ncu-rep --launches gpurun_out/launches_r1.csv \
      --frames-per-launch 16 --tag r1

Writes profiles/ncu_<tag>.md (per-kernel key metrics of the --set full capture, and the per-kernel
share of device time from the launch list) and profiles/ncu_traffic.json (DRAM bytes per launch of
K2 / K1, read by bench.py for the roofline "traffic" field)."""
from __future__ import annotations

import argparse
import csv
import io
import json
import os
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = [
    ("gpu__time_duration.sum", "duration (ns)"),
    ("dram__bytes_read.sum", "DRAM read (B)"),
    ("dram__bytes_write.sum", "DRAM write (B)"),
    ("lts__t_bytes.sum", "L2 bytes (B)"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smem wavefronts"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed", "smem pipe % peak"),
    ("sm__inst_executed.sum", "warp instructions"),
    ("sm__inst_issued.avg.pct_of_peak_sustained_active", "issue slots % (active)"),
    ("smsp__thread_inst_executed_per_inst_executed.ratio", "threads / instruction (SIMT eff.)"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM throughput %"),
    ("gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed", "memory throughput %"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__grid_size", "grid"),
    ("smsp__cycles_active.avg", "SMSP active cycles"),
]


def raw(rep: str):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, data = rows[0], rows[1], rows[2:]
    return [dict(zip(hdr, r)) for r in data], dict(zip(hdr, units))


def num(v):
    try:
        return float(str(v).replace(",", ""))
    except ValueError:
        return None


def launches(path: str):
    rows = list(csv.reader(open(path)))
    for i, r in enumerate(rows):
        if "Kernel Name" in r:
            hdr = r
            data = rows[i + 1:]
            break
    idx = {h: j for j, h in enumerate(hdr)}
    agg = {}
    for r in data:
        if len(r) < len(hdr) or r[idx["Metric Name"]] != "gpu__time_duration.sum":
            continue
        k = r[idx["Kernel Name"]].split("(")[0]
        a = agg.setdefault(k, [0, 0.0])
        a[0] += 1
        a[1] += num(r[idx["Metric Value"]]) or 0.0
    return agg


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--full", required=True)
    ap.add_argument("--launches")
    ap.add_argument("--frames-per-launch", type=int, default=16)
    ap.add_argument("--tag", default="r1")
    ap.add_argument("--l2", help="ncu --metrics lts__t_bytes.sum,... --csv log: per-kernel L2 bytes (first launch)")
    a = ap.parse_args()
    kernels, units = raw(a.full)
    lines = [f"# ncu summary ({a.tag})", "",
             f"`ncu --set full --clock-control none --import-source on` of `bench.py --frames {a.frames_per_launch}` "
             f"(one K2 launch = {a.frames_per_launch} 1080p frames). ncu flushes caches before each replayed "
             "kernel, so DRAM bytes are cold-cache upper bounds.", ""]
    traffic = {}
    seen = set()
    for k in kernels:
        name = k.get("Kernel Name", "?").split("(")[0]
        lines.append(f"## {name}")
        lines.append("")
        lines.append("| metric | value |")
        lines.append("|---|---|")
        for key, label in KEYS:
            if key in k:
                lines.append(f"| {label} (`{key}`) | {k[key]} {units.get(key, '')} |")
        lines.append("")
        def scaled(key):
            v = num(k.get(key)) or 0.0
            return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(units.get(key, "byte"), 1)
        dr = scaled("dram__bytes_read.sum") + scaled("dram__bytes_write.sum")
        l2 = scaled("lts__t_bytes.sum")
        # per-launch DRAM / L2 bytes of each kernel (first capture of each), K1 summed as "k1"
        short = name.split("<")[0].replace("void ", "").strip()
        fam = "k1" if any(t in short for t in ("k_marg", "k_carry", "k_corner", "k_tile")) else short
        if name not in seen:
            seen.add(name)
            t = traffic.setdefault(fam, {"dram_bytes_per_launch": 0.0, "l2_bytes_per_launch": 0.0,
                                         "frames_per_launch": a.frames_per_launch})
            t["dram_bytes_per_launch"] += dr
            t["l2_bytes_per_launch"] += l2
    if a.l2:
        rows = list(csv.reader(open(a.l2)))
        for i, r in enumerate(rows):
            if "Kernel Name" in r:
                hdr, data = r, rows[i + 1:]
                break
        idx = {h: j for j, h in enumerate(hdr)}
        first = {}
        for r in data:
            if len(r) < len(hdr):
                continue
            name = r[idx["Kernel Name"]].split("(")[0].replace("void ", "").split("<")[0].replace("fdk::", "").strip()
            fam = "k1" if any(t in name for t in ("k_marg", "k_tile")) else name
            key = (name, r[idx["ID"]])
            first.setdefault(name, r[idx["ID"]])
            if first[name] != r[idx["ID"]]:
                continue
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(r[idx["Metric Unit"]], 1)
            if r[idx["Metric Name"]] == "lts__t_bytes.sum" and fam in traffic:
                traffic[fam]["l2_bytes_per_launch"] += (num(r[idx["Metric Value"]]) or 0.0) * scale
        lines += ["## L2 traffic (`ncu --metrics lts__t_bytes.sum`, first launch of each kernel, bytes)", "",
                  "| kernel | L2 bytes per launch | DRAM bytes per launch |", "|---|---|---|"]
        for fam, t in traffic.items():
            if isinstance(t, dict):
                lines.append(f"| {fam} | {t['l2_bytes_per_launch']:.3e} | {t['dram_bytes_per_launch']:.3e} |")
        lines.append("")
    if a.launches:
        agg = launches(a.launches)
        tot = sum(v[1] for v in agg.values())
        lines += ["## Launch list (`ncu --metrics gpu__time_duration.sum --clock-control none`)", "",
                  "Cold-cache, serialised per-launch times: compare shares, not absolutes.", "",
                  "| kernel | launches | total us | share |", "|---|---|---|---|"]
        for k, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
            lines.append(f"| {k} | {n} | {t / 1e3:.1f} | {100 * t / tot:.1f}% |")
        lines.append("")
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    with open(os.path.join(ROOT, "profiles", f"ncu_{a.tag}.md"), "w") as fh:
        fh.write("\n".join(lines) + "\n")
    with open(os.path.join(ROOT, "profiles", "ncu_traffic.json"), "w") as fh:
        json.dump(traffic, fh, indent=1)
    print("\n".join(lines))
    print(traffic)


if __name__ == "__main__":
    main()
