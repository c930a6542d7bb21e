#!/usr/bin/env python
"""Group the SASS of one kernel in an ncu report into straight-line runs (equal execution counts) and print the
runs that carry the most instructions or stall samples.

    python tools/sass_hotspots.py <report.ncu-rep> <kernel-regex> [min_share]
"""
import csv
import io
import subprocess
import sys


def main():
    rep, kern = sys.argv[1], sys.argv[2]
    min_share = float(sys.argv[3]) if len(sys.argv) > 3 else 0.005
    txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "-k", f"regex:{kern}", "--print-source",
                          "sass"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr = rows[1]
    ia, isrc, ie = hdr.index("Address"), hdr.index("Source"), hdr.index("Instructions Executed")
    ist = hdr.index("Warp Stall Sampling (All Samples)")
    iw, iwi = hdr.index("L1 Wavefronts Shared"), hdr.index("L1 Wavefronts Shared Ideal")
    data = []
    for r in rows[2:]:
        if len(r) < len(hdr):
            continue
        num = lambda v: int(float(v)) if v not in ("", None) else 0
        data.append((r[ia], r[isrc].strip(), num(r[ie]), num(r[ist]), num(r[iw]), num(r[iwi])))
    groups = []
    for a, s, e, st, w, wi in data:
        op = s.split()[0] if s else ""
        if op.startswith("@"):
            op = s.split()[1] if len(s.split()) > 1 else op
        if groups and groups[-1]["e"] == e:
            g = groups[-1]
        else:
            g = {"a": a, "e": e, "n": 0, "st": 0, "w": 0, "wi": 0, "ops": []}
            groups.append(g)
        g["n"] += 1
        g["st"] += st
        g["w"] += w
        g["wi"] += wi
        g["ops"].append(op)
    tot = sum(d[2] for d in data)
    stt = sum(d[3] for d in data) or 1
    print(f"total instructions {tot:,}  stall samples {stt:,}")
    for g in groups:
        ins = g["n"] * g["e"]
        if ins / tot >= min_share or g["st"] / stt >= min_share:
            wf = f" wf={g['w']/1e6:.2f}M/{g['wi']/1e6:.2f}M" if g["w"] else ""
            print(f"{g['a'][-5:]} x{g['e']:>8} n={g['n']:>3} instr={ins / tot:6.1%} stall={g['st'] / stt:6.1%}{wf}  "
                  f"{' '.join(g['ops'][:14])}")


if __name__ == "__main__":
    main()
