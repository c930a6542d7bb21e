#!/usr/bin/env python
"""Summarise ncu output into the committed profiles/ evidence.

    python tools/ncu_summary.py launches <launches.csv> > profiles/<round>_launches.md
    python tools/ncu_summary.py full <report.ncu-rep> > profiles/<round>_ncu_full.md
    python tools/ncu_summary.py traffic <report.ncu-rep> <config-name> > profiles/ncu_tile_traffic.json

`launches` reads the CSV of `ncu --metrics gpu__time_duration.sum --clock-control none --csv` (cold-cache,
serialised launches: compare SHARES, not absolute times).  `full` reads an `ncu --set full` report with
`ncu -i ... --page raw --csv` (ncu must be on PATH) and lists, per kernel, the metrics the roofline and DESIGN.md
cite.  `traffic` writes the DRAM bytes per launch of k_tile that bench.py reports as roofline.traffic.
"""
import csv
import io
import json
import subprocess
import sys
from collections import OrderedDict, defaultdict


def _rows(text):
    lines = text.splitlines()
    start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
    return list(csv.reader(io.StringIO("\n".join(lines[start:]))))


def short(name):
    name = name.split("(")[0]
    return name.replace("void ", "").replace("starsim::", "")


def launches(path):
    rows = _rows(open(path).read())
    hdr = rows[0]
    i_name, i_val = hdr.index("Kernel Name"), hdr.index("Metric Value")
    agg = OrderedDict()
    for r in rows[1:]:
        if len(r) <= i_val:
            continue
        k = short(r[i_name])
        agg.setdefault(k, []).append(float(r[i_val].replace(",", "")) / 1e3)
    ours = {k: v for k, v in agg.items() if k.startswith("k_")}
    frames = max(len(v) for k, v in ours.items() if k == "k_tile<8>" or k.startswith("k_tile")) if ours else 1
    tot = sum(sum(v) for v in ours.values())
    out = ["| kernel | launches | mean us/launch | share of our kernels' time |", "|---|---|---|---|"]
    for k, v in ours.items():
        out.append(f"| {k} | {len(v)} | {sum(v) / len(v):.2f} | {sum(v) / tot:.1%} |")
    others = {k: v for k, v in agg.items() if not k.startswith("k_")}
    out.append("")
    out.append("Other launches in the captured window (torch fills/copies of the harness, L2 flush): " +
               ", ".join(f"{k} x{len(v)}" for k, v in others.items()))
    out.append(f"\nFrames in window: {frames}.  Per-launch times are ncu's serialised, cold-cache replays.")
    return "\n".join(out)


METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps active % (achieved occupancy)"),
    ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "FMA pipe %"),
    ("sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", "ALU pipe %"),
    ("sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active", "XU (MUFU) pipe %"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "shared-memory wavefronts"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput %"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
]


def raw(path):
    txt = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = _rows(txt)
    hdr, units = rows[0], rows[1]
    return hdr, units, rows[2:]


def full(path):
    hdr, units, rows = raw(path)
    out = []
    for r in rows:
        d = dict(zip(hdr, r))
        u = dict(zip(hdr, units))
        out.append(f"### {short(d['Kernel Name'])} (ID {d['ID']})\n")
        out.append("| metric | value |\n|---|---|")
        for m, label in METRICS:
            if m in d:
                out.append(f"| {label} (`{m}`) | {d[m]} {u.get(m, '')} |")
        stalls = {k.replace("smsp__average_warps_issue_stalled_", "").replace("_per_issue_active.ratio", ""): v
                  for k, v in d.items() if k.startswith("smsp__average_warps_issue_stalled_")
                  and k.endswith("_per_issue_active.ratio")}
        top = sorted(((float(v), k) for k, v in stalls.items() if v not in ("", "n/a")), reverse=True)[:5]
        out.append(f"| top stall reasons (warps per issue) | " + ", ".join(f"{k} {v:.2f}" for v, k in top) + " |")
        out.append("")
    return "\n".join(out)


def traffic(path, cfg):
    hdr, units, rows = raw(path)
    res = {}
    for r in rows:
        d = dict(zip(hdr, r))
        if "k_tile" not in d["Kernel Name"]:
            continue
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
        u = dict(zip(hdr, units))
        rd = float(d["dram__bytes_read.sum"]) * scale.get(u["dram__bytes_read.sum"], 1)
        wr = float(d["dram__bytes_write.sum"]) * scale.get(u["dram__bytes_write.sum"], 1)
        res = {cfg: {"dram_bytes_per_launch": rd + wr, "read": rd, "write": wr,
                     "kernel": short(d["Kernel Name"]),
                     "warp_instructions": float(d.get("smsp__inst_executed.sum", "nan").replace(",", "")),
                     "issue_active_pct": float(d.get("smsp__issue_active.avg.pct_of_peak_sustained_active",
                                                     "nan").replace(",", "")),
                     "fma_pipe_pct": float(d.get("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
                                                 "nan").replace(",", "")),
                     "duration_ns_ncu": float(d["gpu__time_duration.sum"]) *
                     {"us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6}.get(u["gpu__time_duration.sum"], 1)}}
    return json.dumps(res, indent=1)


if __name__ == "__main__":
    mode = sys.argv[1]
    if mode == "launches":
        print(launches(sys.argv[2]))
    elif mode == "full":
        print(full(sys.argv[2]))
    else:
        print(traffic(sys.argv[2], sys.argv[3]))
