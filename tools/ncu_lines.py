"""Per-source-line instruction / stall attribution from an ncu report (cuda,sass source view).

usage: python tools/ncu_lines.py report.ncu-rep [top] [kernel-substring]
"""
import csv
import io
import subprocess
import sys
from collections import defaultdict


def main(rep, top=30, kfilter=None):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    fname, line, src = "?", None, ""
    inst = defaultdict(float)
    stall = defaultdict(float)
    text = {}
    hdr = None
    keep = kfilter is None
    for r in csv.reader(io.StringIO(out)):
        if not r:
            continue
        if r[0] == "File Path":
            fname = r[1].split("/")[-1]
            continue
        if r[0] == "Function Name":
            keep = kfilter is None or kfilter in r[1]
            continue
        if not keep:
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr is None:
            continue
        if r[0]:
            line = (fname, int(r[0]))
            text[line] = ",".join(r[1:len(r) - len(hdr) + 2])[:90]
            continue
        d = dict(zip(hdr[2:], r[len(r) - len(hdr) + 2:]))
        try:
            inst[line] += float(d.get("Instructions Executed", 0) or 0)
            stall[line] += float(d.get("Warp Stall Sampling (All Samples)", 0) or 0)
        except ValueError:
            pass
    ti, ts = sum(inst.values()) or 1, sum(stall.values()) or 1
    print(f"total warp instructions {ti:.0f}, stall samples {ts:.0f}")
    for k in sorted(inst, key=lambda k: -stall[k])[:top]:
        print(f"{k[0]}:{k[1]:5d} inst {100 * inst[k] / ti:5.1f}% stall {100 * stall[k] / ts:5.1f}%  {text.get(k, '')}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 30, sys.argv[3] if len(sys.argv) > 3 else None)
