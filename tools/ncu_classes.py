"""ncu evidence for every kernel class of one training step.

  run:        python tools/ncu_classes.py run --workload cfg2_vgg5 --out gpurun_out/ncu_cfg2
              (under `ncu --metrics $(python tools/ncu_classes.py metrics) --profile-from-start off
              --clock-control none -o <rep>`: two warm-up steps, then
              cudaProfilerStart, ONE profiled step whose every scope is logged by the engine
              (skipper_profile_records: class, kernels, algorithmic bytes / FLOPs), cudaProfilerStop)
  summarise:  python tools/ncu_classes.py summarise <rep.ncu-rep> <records.json> > profiles/r2_ncu_<cfg>.md
              joins the ncu launch list with the engine's records in launch order (the counts must match)
              and reports per class: launches, ncu time, DRAM bytes (read + write) against the algorithmic
              bytes, tensor-pipe activity, achieved occupancy and the limiting unit; writes
              profiles/traffic.json (DRAM bytes per launch, per class).
"""
import argparse
import collections
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def run(a):
    import torch

    import synth
    from paper_conf_micro_singhslsknnd22_b200 import SkipperNet
    wl = synth.workload(a.workload)
    net = synth.net_config(wl["net"])
    x, y = synth.make_inputs(net, wl["T"], wl["B"])
    m = SkipperNet(net, wl["T"], C=wl["C"], p=wl["p"], mode=a.mode, batch=wl["B"])
    m.set_weights(synth.make_weights(net))
    xd, yd = torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda()
    for _ in range(2):
        m.step(xd, yd, want_loss=False)
    torch.cuda.synchronize()
    m.profile(True)
    torch.cuda.profiler.start()
    m.step(xd, yd, want_loss=False)
    torch.cuda.synchronize()
    torch.cuda.profiler.stop()
    recs = m.profile_records()
    m.profile(False)
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out + "_records.json", "w") as f:
        json.dump({"workload": a.workload, "mode": a.mode, "records": recs}, f)
    print("records", len(recs), "kernels", sum(r[1] for r in recs))


METRICS = {
    "t_us": "gpu__time_duration.sum",
    "dram_rd": "dram__bytes_read.sum",
    "dram_wr": "dram__bytes_write.sum",
    "tensor": "sm__pipe_tensor_subpipe_hmma_cycles_active.avg.pct_of_peak_sustained_active",
    "tc": "sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_active",
    "occ": "sm__warps_active.avg.pct_of_peak_sustained_active",
    "sm": "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "dram_pct": "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "l1": "l1tex__throughput.avg.pct_of_peak_sustained_active",
    "tma": "sm__pipe_tma_cycles_active.avg.pct_of_peak_sustained_active",
    "l2": "lts__throughput.avg.pct_of_peak_sustained_elapsed",
    "issue": "sm__inst_issued.avg.pct_of_peak_sustained_active",
}
SCALE = {"us": 1.0, "usecond": 1.0, "ns": 1e-3, "nsecond": 1e-3, "ms": 1e3, "msecond": 1e3,
         "byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}


def ncu_rows(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    hdr, units, rows = r[0], r[1], r[2:]
    res = []
    for row in rows:
        d = dict(zip(hdr, row))
        u = dict(zip(hdr, units))
        e = {"name": d.get("Kernel Name", "?").split("(")[0], "grid": d.get("Grid Size", "")}
        for k, mname in METRICS.items():
            v = d.get(mname, "")
            try:
                val = float(v.replace(",", ""))
            except ValueError:
                val = float("nan")
            e[k] = val * SCALE.get(u.get(mname, ""), 1.0) if k in ("t_us", "dram_rd", "dram_wr") else val
        res.append(e)
    return res


def summarise(a):
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    rows = ncu_rows(a.rep)
    meta = json.load(open(a.records))
    recs = meta["records"]
    nk = sum(r[1] for r in recs)
    if nk != len(rows):
        raise SystemExit(f"launch count mismatch: engine {nk} kernels, ncu {len(rows)}")
    cls = collections.OrderedDict()
    i = 0
    for name, k, by, fl, _ in recs:
        c = cls.setdefault(name, {"launches": 0, "kernels": collections.Counter(), "t": 0.0, "dram": 0.0, "alg": 0.0,
                                  "flops": 0.0, "tensor_t": 0.0, "occ_t": 0.0, "lim": collections.Counter()})
        c["launches"] += 1
        c["alg"] += by
        c["flops"] += fl
        for r in rows[i:i + k]:
            c["kernels"][r["name"]] += 1
            c["t"] += r["t_us"]
            c["dram"] += r["dram_rd"] + r["dram_wr"]
            tens = r["tensor"] if r["tensor"] == r["tensor"] else r["tc"]   # hmma subpipe counts UTCHMMA
            c["tensor_t"] += (tens if tens == tens else 0.0) * r["t_us"]
            c["occ_t"] += (r["occ"] if r["occ"] == r["occ"] else 0.0) * r["t_us"]
            units = {"DRAM": r["dram_pct"], "L1/TEX": r["l1"], "L2": r["l2"], "SM issue": r["issue"],
                     "tensor": tens, "TMA": r["tma"]}
            units = {u: v for u, v in units.items() if v == v}
            if units:
                top = max(units, key=units.get)
                c["lim"][f"{top} {units[top]:.0f}%"] += r["t_us"]
        i += k
    print(f"ncu --clock-control none (the metrics of `tools/ncu_classes.py metrics`), one {meta['mode'].upper()} training step of {meta['workload']} "
          f"(tools/ncu_classes.py; kernels serialised and cold-cache under replay, so absolute times run long).  "
          f"`alg` = the engine's algorithmic bytes (DESIGN.md §7); `DRAM/alg` > 1.2 flags wasted traffic.  "
          f"HBM peak {peaks['hbm_gbs']:.0f} GB/s, sustained bf16 {peaks['bf16_tflops_sustained']:.0f} TF/s "
          f"(MEASURED_PEAKS.json).\n")
    print("| class | launches | kernels | ncu time (us) | DRAM (MB) | alg (MB) | DRAM/alg | DRAM GB/s (frac) "
          "| alg TF/s (frac) | tensor pipe % | occupancy % | limiter (time-weighted) |")
    print("|---|---|---|---|---|---|---|---|---|---|---|---|")
    traffic = {}
    for name, c in cls.items():
        t = c["t"] or 1e-9
        gbs = c["dram"] / (t * 1e-6) / 1e9
        tfs = c["flops"] / (t * 1e-6) / 1e12
        lim = c["lim"].most_common(1)[0][0] if c["lim"] else "-"
        ks = ", ".join(f"{k.replace('void ', '')[:40]} x{n}" for k, n in c["kernels"].most_common(3))
        flag = " **wasted**" if c["alg"] and c["dram"] > 1.2 * c["alg"] else ""
        print(f"| {name} | {c['launches']} | {ks} | {c['t']:.1f} | {c['dram'] / 1e6:.1f} | {c['alg'] / 1e6:.1f} | "
              f"{(c['dram'] / c['alg'] if c['alg'] else float('nan')):.2f}{flag} | {gbs:.0f} ({gbs / peaks['hbm_gbs']:.2f}) | "
              f"{tfs:.0f} ({tfs / peaks['bf16_tflops_sustained']:.2f}) | {c['tensor_t'] / t:.1f} | {c['occ_t'] / t:.1f} | {lim} |")
        traffic[name] = c["dram"] / max(c["launches"], 1)
    if a.traffic:
        tf = os.path.join(ROOT, "profiles", "traffic.json")
        old = json.load(open(tf)) if os.path.exists(tf) else {}
        old.update({f"{meta['workload']}:{k}": v for k, v in traffic.items()})
        if meta["workload"] == "cfg2_vgg5" and meta["mode"] == "skip":
            old.update(traffic)   # the bench's default workload: unprefixed keys, read by bench.py
        old["_note"] = ("dram__bytes_read.sum + dram__bytes_write.sum per launch of the class (mean over the "
                        "class's launches in one ncu metrics capture of a training step, tools/ncu_classes.py)")
        json.dump(old, open(tf, "w"), indent=1, sort_keys=True)


def main():
    ap = argparse.ArgumentParser()
    sp = ap.add_subparsers(dest="cmd", required=True)
    r = sp.add_parser("run")
    r.add_argument("--workload", default="cfg2_vgg5")
    r.add_argument("--mode", default="skip")
    r.add_argument("--out", required=True)
    s = sp.add_parser("summarise")
    s.add_argument("rep")
    s.add_argument("records")
    s.add_argument("--traffic", action="store_true")
    sp.add_parser("metrics")
    a = ap.parse_args()
    if a.cmd == "metrics":
        print(",".join(METRICS.values()))
    else:
        run(a) if a.cmd == "run" else summarise(a)


if __name__ == "__main__":
    main()
