"""Summarise an ncu --metrics gpu__time_duration.sum launch list: one training step's kernels."""
import csv, collections, re, sys

def load(path):
    lines = [l for l in open(path) if l.startswith('"')]
    rows = list(csv.DictReader(lines))
    return [(r["Kernel Name"], r["Grid Size"], float(r["Metric Value"])) for r in rows
            if r["Metric Name"] == "gpu__time_duration.sum"]

def short(n):
    n = re.sub(r"\(.*", "", n)
    return n.replace("sk::", "")

if __name__ == "__main__":
    rows = load(sys.argv[1])
    # one step = launches between two consecutive adam_kernel groups; take the last complete step
    idx = [i for i, r in enumerate(rows) if short(r[0]).startswith("adam_kernel")]
    # steps end after the last adam+transpose of a step; group adam runs
    ends = [i for j, i in enumerate(idx) if j + 1 == len(idx) or idx[j + 1] - i > 5]
    if len(ends) >= 2:
        a, b = ends[-2] + 1, ends[-1] + 1
        while b < len(rows) and short(rows[b][0]).startswith(("transpose", "cast_pad")):
            b += 1
        while a < len(rows) and short(rows[a][0]).startswith(("transpose", "cast_pad")):
            a += 1
        rows = rows[a:b]
    tot = sum(r[2] for r in rows)
    agg = collections.defaultdict(lambda: [0, 0.0])
    for n, g, t in rows:
        k = short(n)
        agg[k][0] += 1
        agg[k][1] += t
    print(f"launches {len(rows)}  total {tot/1e6:.3f} ms (serialised, cold)")
    for k, (c, t) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        print(f"{k:60s} {c:5d} {t/1e6:8.3f} ms {100*t/tot:5.1f}%")
    if len(sys.argv) > 2:
        for n, g, t in rows:
            print(f"{short(n)[:40]:40s} {g:16s} {t/1e3:9.1f} us")
