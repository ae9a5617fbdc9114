"""Summarise `ncu --set full` reports into a markdown table (for profiles/).

usage: python tools/ncu_summary.py report.ncu-rep [...] > profiles/<name>.md
"""
import csv
import io
import subprocess
import sys

METRICS = [
    ("gpu__time_duration.sum", "us", 1.0),
    ("dram__bytes_read.sum", "MB", 1.0),
    ("dram__bytes_write.sum", "MB", 1.0),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "% DRAM", 1.0),
    ("sm__pipe_tensor_subpipe_hmma_cycles_active.avg.pct_of_peak_sustained_active", "% tensor pipe", 1.0),
    ("sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_active", "% TC pipe", 1.0),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "% SM", 1.0),
    ("lts__t_bytes.sum", "L2 bytes", 1.0),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "% warps active", 1.0),
    ("launch__registers_per_thread", "regs", 1.0),
]


def rows_of(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    if len(r) < 3:
        return [], [], []
    return r[0], r[1], r[2:]


def main(reps):
    print("| report | kernel | grid | " + " | ".join(m[0].split(".")[0] + f" ({m[1]})" for m in METRICS) + " |")
    print("|" + "---|" * (3 + len(METRICS)))
    for rep in reps:
        hdr, units, rows = rows_of(rep)
        for r in rows:
            d = dict(zip(hdr, r))
            u = dict(zip(hdr, units))
            name = d.get("Kernel Name", "?").split("(")[0][:48]
            vals = []
            for m, _, _ in METRICS:
                v = d.get(m, "")
                unit = u.get(m, "")
                vals.append(f"{v} {unit}".strip())
            print(f"| {rep.split('/')[-1]} | {name} | {d.get('Grid Size', '')} | " + " | ".join(vals) + " |")


if __name__ == "__main__":
    main(sys.argv[1:])
