#!/usr/bin/env python
"""Benchmark: SNN train samples/s and peak HBM (Skipper vs full BPTT), VGG-CIFAR.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload cfg2_vgg5] [--mode skip]
    python bench.py --impl reference ...      (the CPU oracle arm)

One step = one full training iteration through the C ABI (skipper_step): first
forward pass with checkpoints + SAM, loss, SST/keep mask, per-segment recompute
and backward, gradient allreduce (N>1), Adam.  Inputs resident in HBM; L2 is
flushed (512 MB write) between timed steps; each step timed with CUDA events on
the library's stream; max over ranks.  Rank 0 prints one JSON line.
"""
from __future__ import annotations

import os

_CORES = len(os.sched_getaffinity(0))
for _v in ("OMP_NUM_THREADS", "OPENBLAS_NUM_THREADS", "MKL_NUM_THREADS"):
    os.environ.setdefault(_v, str(_CORES))

import argparse  # noqa: E402
import json  # noqa: E402
import statistics  # noqa: E402
import subprocess  # noqa: E402
import sys  # noqa: E402
import tempfile  # noqa: E402
import time  # noqa: E402

import numpy as np  # noqa: E402

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synth  # noqa: E402

METRIC = "SNN train samples/s and peak HBM GB vs T (Skipper vs full BPTT), VGG-CIFAR"
UNIT = "samples/s"


def load_peaks():
    """MEASURED_PEAKS.json (driver-written); else this pool's measured values recorded earlier in the
    round (profiles/measured_peaks_r1.json); else the profiling guide's fallback."""
    for fn, src in (("MEASURED_PEAKS.json", "measured"),
                    (os.path.join("profiles", "measured_peaks_r1.json"), "measured (profiles/measured_peaks_r1.json)")):
        try:
            with open(os.path.join(ROOT, fn)) as f:
                d = json.load(f)
            return {"hbm_gbs": d["hbm_gbs"], "bf16_tflops": d["bf16_tflops"],
                    "bf16_tflops_sustained": d["bf16_tflops_sustained"], "source": src}
        except Exception:  # noqa: BLE001
            continue
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0, "source": "fallback"}


def workload_config(args):
    wl = synth.workload(args.workload)
    net = synth.net_config(wl["net"])
    if args.T:
        wl["T"] = args.T
    if args.batch:
        wl["B"] = args.batch
    if args.C:
        wl["C"] = args.C
    if args.p is not None:
        wl["p"] = args.p
    return wl, net


def describe(net):
    parts = []
    for L in net["layers"]:
        if L["kind"] == "conv":
            parts.append(f"conv{L['cin']}-{L['cout']}@{L['h']}" + ("p" if L["pool"] else "")
                         + ("s2" if L.get("stride", 1) == 2 else "") + (f"+r{L['res']}" if "res" in L else ""))
        elif L["kind"] == "fc":
            parts.append(f"fc{L['cin']}-{L['cout']}")
        else:
            parts.append(("gap-" if L.get("gap") else "") + f"readout{L['cin']}-{L['cout']}")
    return " ".join(parts)


# ------------------------------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 50 ms during the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap,memory.used")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.f = None

    def start(self):
        try:
            self.f = tempfile.TemporaryFile(mode="w+")
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "50"], stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:  # noqa: BLE001
            self.proc = None

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:  # noqa: BLE001
            self.proc.kill()
        self.f.seek(0)
        rows = [r.split(",") for r in self.f.read().strip().splitlines() if r.strip()]
        sm, mx, reasons, mem = [], None, set(), []
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            try:
                sm.append(float(r[0]))
                mx = float(r[1])
                for nm, v in zip(names, r[4:8]):
                    if v.strip().lower() == "active":
                        reasons.add(nm)
                mem.append(float(r[8]))
            except (ValueError, IndexError):
                continue
        loaded = [v for v in sm if mx and v > 0.5 * mx] or sm
        self.mem_used_mib_max = max(mem) if mem else None
        return {"sm_mhz": statistics.median(loaded) if loaded else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------------------------- oracle arms
def oracle_samples_per_s(net, wl, mode, B_s, steps, warmup=0):
    """Time the CPU oracle (as it stands) on a bounded sample: B_s samples, full T."""
    from oracle import StepConfig, train_step
    x, y = synth.make_inputs(net, wl["T"], B_s, seed=1)
    W = synth.make_weights(net)
    cfg = StepConfig(T=wl["T"], C=wl["C"], p=wl["p"], mode=mode, global_batch=B_s)
    for _ in range(warmup):
        train_step(net, W, x, y, cfg)
    times = []
    for _ in range(steps):
        t0 = time.perf_counter()
        train_step(net, W, x, y, cfg)
        times.append(time.perf_counter() - t0)
    tot = sum(times)
    return B_s * steps / tot, 1000.0 * tot / steps


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    wl, net = workload_config(args)
    B_s = args.ref_batch
    val, ms = oracle_samples_per_s(net, wl, args.mode, B_s, args.steps, args.warmup)
    sample = f"B={B_s} of {wl['B']} per step, full T={wl['T']}, C={wl['C']}, p={wl['p']}, mode={args.mode}"
    line = {
        "impl": "reference", "metric": METRIC, "value": val, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f32 forward / f64 backward", "data": "synthetic",
        "config": config_block(args, wl, net),
        "cpu_baseline": {"value": val, "unit": UNIT, "cores": _CORES, "kind": "oracle", "sample": sample},
        "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def config_block(args, wl, net):
    return {"workload": args.workload, "net": describe(net), "T": wl["T"], "per_gpu_batch": wl["B"],
            "global_batch": wl["B"] * args.gpus, "C": wl["C"], "p": wl["p"], "mode": args.mode,
            "parallelism": f"dp{args.gpus}", "l2": "flushed between timed steps (512 MB write)",
            "inputs": ("DVS-Gesture-shaped event frames (2x128x128, moving blob, burst envelope)"
                       if net["input"][0] == "dvs" else "Poisson rate-coded CIFAR-shaped frames")
                      + ", seeded; grid-quantised random weights"}


# ------------------------------------------------------------------------------------- GPU arm
def library_id():
    """sha256 prefix and mtime of the libskipper.so this run loaded (stale-binary check)."""
    import hashlib
    lib = os.path.join(ROOT, "paper_conf_micro_singhslsknnd22_b200", "libskipper.so")
    with open(lib, "rb") as f:
        h = hashlib.sha256(f.read()).hexdigest()[:16]
    return {"file": "libskipper.so", "sha256_16": h,
            "mtime": time.strftime("%Y-%m-%dT%H:%M:%SZ", time.gmtime(os.path.getmtime(lib)))}


_INPUT_CACHE = {}


def cached_inputs(net, T, B, seed):
    """Seeded inputs; frames are prefix-consistent in T (synth draws them in t order), so the longest
    sequence generated so far for (net, B, seed) is reused by slicing."""
    key = (json.dumps(net["input"]), net["layers"][-1]["cout"], B, seed)
    hit = _INPUT_CACHE.get(key)
    if hit is None or hit[0].shape[0] < T:
        _INPUT_CACHE.clear()
        hit = synth.make_inputs(net, T, B, seed=seed)
        _INPUT_CACHE[key] = hit
    return np.ascontiguousarray(hit[0][:T]), hit[1]


def run_mode(torch, dist, args, wl, net, mode, rank, world, local_rank, profile=False, e2e=False, steps=None,
             warmup=None):
    steps = steps or args.steps
    warmup = warmup or args.warmup
    from paper_conf_micro_singhslsknnd22_b200 import SkipperNet
    T, B, C, p = wl["T"], wl["B"], wl["C"], wl["p"]
    x, y = cached_inputs(net, T, B, seed=1 + 1000 * rank)
    W = synth.make_weights(net)
    m = SkipperNet(net, T, C=C, p=p, mode=mode, batch=B, global_batch=B * world, group=args.group)
    m.set_weights(W)
    if world > 1:
        obj = [m.comm_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        m.comm_init(obj[0], rank, world)
    xd = torch.from_numpy(x).cuda()
    yd = torch.from_numpy(y).cuda()
    flush = torch.empty(512 * 1024 * 1024, dtype=torch.uint8, device="cuda")
    for _ in range(warmup):
        m.step(xd, yd, want_loss=False)
    torch.cuda.synchronize()
    m.reset_peak()
    torch.cuda.reset_peak_memory_stats()
    clocks = ClockSampler(local_rank)
    clocks.start() if profile else None
    launches0 = m.launch_count()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    stream = torch.cuda.current_stream()
    evs = []
    for _ in range(steps):
        flush.zero_()
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record(stream)
        m.step(xd, yd, want_loss=False)
        b.record(stream)
        evs.append((a, b))
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clk = clocks.stop() if profile else None
    nvml_used = getattr(clocks, "mem_used_mib_max", None) if profile else None
    ms_list = [a.elapsed_time(b) for a, b in evs]
    tot = torch.tensor([sum(ms_list)], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(tot, op=dist.ReduceOp.MAX)
    total_ms = float(tot.item())
    launches = m.launch_count() - launches0
    prof = None
    if profile:
        # kernel-class attribution: the same K steps again with every launch bracketed by CUDA
        # events on the library stream (kept out of the headline timing: the event records add
        # host work per launch)
        m.profile(True)
        for _ in range(args.steps):
            flush.zero_()
            m.step(xd, yd, want_loss=False)
        prof = m.profile_read()
        m.profile(False)
    peak_lib = m.mem_stats()[1]
    peak_torch = torch.cuda.max_memory_allocated()
    peak_reserved = torch.cuda.max_memory_reserved()
    loss = m.loss()
    res = {"total_ms": total_ms, "ms_list": ms_list, "launches": launches, "prof": prof, "clocks": clk,
           "peak_lib": peak_lib, "peak_torch": peak_torch, "peak_reserved": peak_reserved, "nvml_used": nvml_used,
           "loss": loss,
           "kept_fraction": float(m.keep_mask().mean())}
    if e2e:
        xh = torch.from_numpy(x).pin_memory()
        yh = torch.from_numpy(y).pin_memory()
        xn, yn = xh.numpy(), yh.numpy()
        for _ in range(2):
            m.step_host(xn, yn)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        ts = []
        for _ in range(args.steps):
            flush.zero_()
            torch.cuda.synchronize()
            a = torch.cuda.Event(enable_timing=True)
            b = torch.cuda.Event(enable_timing=True)
            a.record(stream)
            m.step_host(xn, yn)       # H2D of x/labels, the step, D2H of s_t and the loss
            b.record(stream)
            ts.append((a, b))
        torch.cuda.synchronize()
        e2e_ms = torch.tensor([sum(a.elapsed_time(b) for a, b in ts)], dtype=torch.float64, device="cuda")
        if world > 1:
            dist.all_reduce(e2e_ms, op=dist.ReduceOp.MAX)
        res["e2e_ms"] = float(e2e_ms.item())
        res["h2d"] = int(x.nbytes + y.nbytes)
        res["d2h"] = int(4 + 8 * T)
        if net["input"][0] != "dvs":
            # the user call from intensities: H2D of the images, rates and labels, on-device Poisson
            # encoding (Philox), the step, D2H of the loss
            img = np.random.default_rng(1 + 1000 * rank).random((B,) + tuple(x.shape[2:]), dtype=np.float32)
            imh = torch.from_numpy(img).pin_memory()
            rth = torch.from_numpy(synth.envelope(np.arange(T)).astype(np.float32)).pin_memory()
            imn, rtn = imh.numpy(), rth.numpy()
            for _ in range(2):
                m.step_host_encoded(imn, rtn, 7, yn)
            torch.cuda.synchronize()
            if world > 1:
                dist.barrier()
            ts = []
            for _ in range(args.steps):
                flush.zero_()
                torch.cuda.synchronize()
                a = torch.cuda.Event(enable_timing=True)
                b = torch.cuda.Event(enable_timing=True)
                a.record(stream)
                m.step_host_encoded(imn, rtn, 7, yn)
                b.record(stream)
                ts.append((a, b))
            torch.cuda.synchronize()
            enc_ms = torch.tensor([sum(a.elapsed_time(b) for a, b in ts)], dtype=torch.float64, device="cuda")
            if world > 1:
                dist.all_reduce(enc_ms, op=dist.ReduceOp.MAX)
            res["e2e_enc_ms"] = float(enc_ms.item())
            res["h2d_enc"] = int(img.nbytes + 4 * T + y.nbytes)
    m.close()
    del flush
    torch.cuda.empty_cache()
    return res


def roofline(prof, peaks, steps):
    """Dominant kernel class of the step and its achieved fraction of the B200 roofline."""
    total = sum(v["ms"] for v in prof.values()) or 1.0
    breakdown = {}
    ridge = peaks["bf16_tflops_sustained"] * 1e12 / (peaks["hbm_gbs"] * 1e9)
    for k, v in prof.items():
        if v["launches"] == 0:
            continue
        per_ms = v["ms"] / v["launches"]
        gbs = v["bytes"] / v["launches"] / (per_ms * 1e-3) / 1e9
        tfs = v["flops"] / v["launches"] / (per_ms * 1e-3) / 1e12 if v["flops"] else 0.0
        tensor = k.startswith("gemm") and v["flops"] / max(v["bytes"], 1) > ridge
        breakdown[k] = {"ms_per_step": v["ms"] / steps, "share": v["ms"] / total, "launches_per_step": v["launches"] / steps,
                        "GB/s": gbs, "TFLOP/s": tfs,
                        "frac": (tfs / peaks["bf16_tflops_sustained"]) if tensor else (gbs / peaks["hbm_gbs"]),
                        "bound": "tensor" if tensor else "hbm"}
    # step roofline: every kernel class at max(FLOP-time, byte-time) of its algorithmic
    # work, summed (no overlap credit) -> the time a roofline-speed implementation of this schedule takes
    roof_ms = 0.0
    for k, v in prof.items():
        if v["launches"] == 0:
            continue
        t_f = v["flops"] / (peaks["bf16_tflops_sustained"] * 1e12) if k.startswith("gemm") or k.startswith("layer0") else 0.0
        t_b = v["bytes"] / (peaks["hbm_gbs"] * 1e9)
        roof_ms += 1e3 * max(t_f, t_b) / steps
    dom = max(breakdown, key=lambda k: breakdown[k]["ms_per_step"])
    d = breakdown[dom]
    traffic = None
    tf = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tf):
        try:
            traffic = json.load(open(tf)).get(dom)
        except Exception:  # noqa: BLE001
            traffic = None
    if d["bound"] == "tensor":
        rf = {"bound": "tensor", "achieved": d["TFLOP/s"], "peak": peaks["bf16_tflops_sustained"], "unit": "TFLOP/s",
              "frac": d["frac"], "traffic": traffic, "kernel": dom}
    else:
        rf = {"bound": "hbm", "achieved": d["GB/s"], "peak": peaks["hbm_gbs"], "unit": "GB/s", "frac": d["frac"],
              "traffic": traffic, "kernel": dom}
    rf["peak_source"] = peaks["source"] + (" (sustained bf16)" if d["bound"] == "tensor" else " (copy bandwidth)")
    return rf, breakdown, roof_ms


def sqrt_divisor(T, L_n):
    """C for the C ~ sqrt(T) leg of cfg 5: the divisor of T nearest sqrt(T) whose segment length T/C exceeds
    the layer count - Eq.3's minimum of C + T/C."""
    cands = [C for C in range(1, T + 1) if T % C == 0 and T // C > L_n]
    return min(cands, key=lambda C: (abs(C - T ** 0.5), C))


def sweep_sqrt_c(torch, dist, args, rank, world, local_rank):
    """cfg 5, C ~ sqrt(T) leg: peak HBM and throughput of CKPT and SKIP with C chosen per T as above; the stored
    state is O(C + T/C) = O(sqrt(T)) (Eq.3 / Eq.6), so peak HBM should grow like sqrt(T), not T."""
    w5 = synth.workload("cfg3_vgg11")
    net5 = synth.net_config(w5["net"])
    L_n = len(net5["layers"])
    out = {}
    for T in [int(v) for v in args.t_sweep_vgg11.split(",") if v]:
        C = sqrt_divisor(T, L_n)
        w2 = dict(w5, T=T, C=C)
        row = {"C": C}
        for mode in ("skip", "ckpt"):
            try:
                r = run_mode(torch, dist, args, w2, net5, mode, rank, world, local_rank, steps=3, warmup=3)
                row[mode] = {"samples_per_s": w2["B"] * world * 3 / (r["total_ms"] / 1e3),
                             "peak_hbm_gb": r["peak_lib"] / 1e9}
            except Exception as e:  # noqa: BLE001
                row[mode] = {"error": str(e)[:120]}
        out[str(T)] = row
    Ts = sorted(int(t) for t in out)
    for mode in ("skip", "ckpt"):
        try:   # growth exponent of the peak between the smallest and largest T (1 = linear, 0.5 = sqrt)
            a, b = out[str(Ts[0])][mode]["peak_hbm_gb"], out[str(Ts[-1])][mode]["peak_hbm_gb"]
            out[f"{mode}_growth_exponent"] = float(np.log(b / a) / np.log(Ts[-1] / Ts[0]))
        except Exception:  # noqa: BLE001
            pass
    return out


def max_t_search(torch, dist, args, rank, world, local_rank, sweep11):
    """cfg 5 / Fig. 14: the largest T (multiple of 100) each mode trains at C = 5, p = 50 within a
    memory budget - the A100's 80 GB and this device's whole HBM.  Peak HBM at fixed C is affine in T, so T_max is
    predicted from the two largest T of the C = 5 sweep and then CHECKED by training steps: bisection (multiples
    of 100) between the largest sweep T that fit and the prediction, each probe one step whose measured peak must
    stay within the budget (an allocation failure counts as not fitting)."""
    w5 = synth.workload("cfg3_vgg11")
    net5 = synth.net_config(w5["net"])
    total = torch.cuda.mem_get_info()[1]
    budgets = {"80GB": 80e9, "device_hbm": float(total)}
    out = {"budgets_gb": {k: v / 1e9 for k, v in budgets.items()}, "C": 5, "p": w5["p"],
           "peak": "library allocator high-water mark (the stored-state + workspace bytes of the step)"}
    for bname, budget in budgets.items():
        res = {}
        for mode in ("full", "ckpt", "skip"):
            pts = sorted((int(T), row[mode]["peak_hbm_gb"] * 1e9) for T, row in sweep11.items()
                         if "peak_hbm_gb" in row.get(mode, {}))
            if len(pts) < 2:
                res[mode] = {"error": "fewer than two sweep points"}
                continue
            (t1, p1), (t2, p2) = pts[-2], pts[-1]
            slope = (p2 - p1) / (t2 - t1)
            Tm = int((t2 + (budget - p2) / slope) // 100 * 100)
            entry = {"predicted_T_max": Tm}

            def fits(T):
                try:
                    r = run_mode(torch, dist, args, dict(w5, T=T, C=5), net5, mode, rank, world, local_rank, steps=1,
                                 warmup=1)
                except Exception as e:  # noqa: BLE001
                    entry.setdefault("failed", []).append([T, str(e)[:80]])
                    return None
                if r["peak_lib"] > budget:
                    entry.setdefault("over_budget", []).append([T, r["peak_lib"] / 1e9])
                    return None
                return r
            # bisection on multiples of 100 between the largest sweep T known to fit and the prediction
            lo, hi = (t2 // 100) * 100 if p2 <= budget else 0, Tm + 100
            best = None
            r = fits(Tm) if Tm >= 100 else None
            if r is not None:
                lo, best = Tm, (Tm, r)
            else:
                hi = Tm
            for _ in range(6):
                if hi - lo <= 100:
                    break
                mid = (lo + hi) // 200 * 100
                r = fits(mid)
                if r is not None:
                    lo, best = mid, (mid, r)
                else:
                    hi = mid
            if best is None and lo >= 100 and lo == (t2 // 100) * 100:
                best = (lo, None)
            if best is not None:
                entry["T_max"] = best[0]
                if best[1] is not None:
                    entry.update({"peak_hbm_gb": best[1]["peak_lib"] / 1e9,
                                  "samples_per_s": w5["B"] * world / (best[1]["total_ms"] / 1e3)})
            res[mode] = entry
        for mode in ("ckpt", "skip"):
            try:
                res[f"{mode}_over_full"] = res[mode]["T_max"] / res["full"]["T_max"]
            except Exception:  # noqa: BLE001
                pass
        out[bname] = res
    out["paper"] = "A100 80 GB, VGG11/CIFAR100: BPTT T_max 200, checkpointed 4.5x (T=900), Skipper 9x (T=1800)"
    return out


def run_ours(args):
    import torch
    import torch.distributed as dist
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.gpus != world and world > 1:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world}")
    torch.cuda.set_device(local_rank)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    import __graft_entry__
    if rank == 0:
        __graft_entry__.build()   # incremental (mtime-checked): a no-op unless csrc changed
    if world > 1:
        dist.barrier()
    wl, net = workload_config(args)
    peaks = load_peaks()
    main = run_mode(torch, dist, args, wl, net, args.mode, rank, world, local_rank, profile=True, e2e=True)
    compare = {}
    if not args.no_compare:
        for mode in ("full", "ckpt", "tbptt"):   # tbptt: the paper's comparison algorithm (Sec. III-C), t' = T/C
            if mode == args.mode:
                continue
            try:
                r = run_mode(torch, dist, args, wl, net, mode, rank, world, local_rank)
                compare[mode] = {"samples_per_s": wl["B"] * world * args.steps / (r["total_ms"] / 1e3),
                                 "ms_per_step": r["total_ms"] / args.steps, "peak_hbm_gb": r["peak_lib"] / 1e9}
            except Exception as e:  # noqa: BLE001
                compare[mode] = {"error": str(e)[:200]}
        # backward groups (skipper_config.group): G segments per layer-major backward pass, G x the segment arena
        if args.mode in ("skip", "ckpt"):
            for G in sorted({2, wl["C"]} - {args.group}):
                try:
                    a2 = argparse.Namespace(**dict(vars(args), group=G))
                    r = run_mode(torch, dist, a2, wl, net, args.mode, rank, world, local_rank)
                    compare[f"{args.mode}_group{G}"] = {
                        "samples_per_s": wl["B"] * world * args.steps / (r["total_ms"] / 1e3),
                        "ms_per_step": r["total_ms"] / args.steps, "peak_hbm_gb": r["peak_lib"] / 1e9}
                except Exception as e:  # noqa: BLE001
                    compare[f"{args.mode}_group{G}"] = {"error": str(e)[:200]}
    # peak HBM and throughput vs T (the metric's "vs T"): Skipper vs full BPTT, segment length S fixed
    t_sweep = {}
    if not args.no_compare and args.t_sweep:
        S = wl["T"] // wl["C"]
        for T in [int(v) for v in args.t_sweep.split(",") if v]:
            if T % S:
                continue
            w2 = dict(wl, T=T, C=T // S)
            row = {}
            for mode in ("skip", "full"):
                try:
                    r = run_mode(torch, dist, args, w2, net, mode, rank, world, local_rank, steps=3, warmup=3)
                    row[mode] = {"samples_per_s": w2["B"] * world * 3 / (r["total_ms"] / 1e3),
                                 "peak_hbm_gb": r["peak_lib"] / 1e9}
                except Exception as e:  # noqa: BLE001
                    row[mode] = {"error": str(e)[:160]}
            t_sweep[str(T)] = row
    # the other BASELINE.json configs at N GPUs (per-GPU batch fixed): cfg 3 VGG-11, cfg 4 ResNet-DVS
    other = {}
    if not args.no_compare and args.workloads:
        for name in [w for w in args.workloads.split(",") if w]:
            w2 = synth.workload(name)
            net2 = synth.net_config(w2["net"])
            row = {"net": describe(net2), "T": w2["T"], "per_gpu_batch": w2["B"], "C": w2["C"], "p": w2["p"]}
            for mode in ("skip", "ckpt", "full"):
                try:
                    r = run_mode(torch, dist, args, w2, net2, mode, rank, world, local_rank, steps=5, warmup=3)
                    row[mode] = {"samples_per_s": w2["B"] * world * 5 / (r["total_ms"] / 1e3),
                                 "ms_per_step": r["total_ms"] / 5, "peak_hbm_gb": r["peak_lib"] / 1e9,
                                 "kept_fraction": r["kept_fraction"]}
                except Exception as e:  # noqa: BLE001
                    row[mode] = {"error": str(e)[:160]}
            other[name] = row
    # cfg 5: VGG-11 T sweep at per-GPU B = 128, C = 5, p = 50 (Fig. 14 setting): throughput and peak HBM
    # per mode; FULL stops fitting in HBM as T grows (reported as its allocation error)
    sweep11 = {}
    if not args.no_compare and args.t_sweep_vgg11:
        w5 = synth.workload("cfg3_vgg11")
        net5 = synth.net_config(w5["net"])
        for T in [int(v) for v in args.t_sweep_vgg11.split(",") if v]:
            w2 = dict(w5, T=T, C=5)
            row = {}
            for mode in ("skip", "ckpt", "full"):
                try:
                    r = run_mode(torch, dist, args, w2, net5, mode, rank, world, local_rank, steps=3, warmup=3)
                    row[mode] = {"samples_per_s": w2["B"] * world * 3 / (r["total_ms"] / 1e3),
                                 "peak_hbm_gb": r["peak_lib"] / 1e9}
                except Exception as e:  # noqa: BLE001
                    row[mode] = {"error": str(e)[:120]}
            sweep11[str(T)] = row
    sqrt_leg, max_t = {}, {}
    if not args.no_compare and args.t_sweep_vgg11:
        sqrt_leg = sweep_sqrt_c(torch, dist, args, rank, world, local_rank)
        if args.max_t:
            max_t = max_t_search(torch, dist, args, rank, world, local_rank, sweep11)
    if rank != 0:
        if world > 1:
            dist.barrier()
            dist.destroy_process_group()
        return
    gb = wl["B"] * world
    value = gb * args.steps / (main["total_ms"] / 1e3)
    rf, breakdown, roof_ms = roofline(main["prof"], peaks, args.steps)
    cfg = config_block(args, wl, net)
    cfg["peak_hbm_gb"] = main["peak_lib"] / 1e9
    cfg["peak_torch_allocated_gb"] = main["peak_torch"] / 1e9
    # the paper's three memory readings: max_memory_allocated, max_memory_reserved, and the
    # overall device memory NVML reports (nvidia-smi memory.used, max over the 50 ms samples of the timed
    # region: includes the CUDA context, cuBLAS/NCCL workspaces, and the bench's 512 MB L2-flush buffer)
    cfg["peak_torch_reserved_gb"] = main["peak_reserved"] / 1e9
    cfg["nvml_used_gb_max"] = main["nvml_used"] * 1.048576e-3 if main["nvml_used"] else None
    cfg["kept_fraction"] = main["kept_fraction"]
    cfg["compare"] = compare
    cfg["library"] = library_id()
    if t_sweep:
        cfg["t_sweep"] = t_sweep
    if other:
        cfg["other_workloads"] = other
    if sweep11:
        cfg["t_sweep_vgg11_cfg5"] = sweep11
    if sqrt_leg:
        cfg["t_sweep_vgg11_cfg5_c_sqrt_t"] = sqrt_leg
    if max_t:
        cfg["max_t_vgg11_cfg5"] = max_t
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": main["total_ms"] / args.steps, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "bf16", "data": "synthetic", "config": cfg,
        "roofline": rf,
        "e2e": ({"value": gb * args.steps / (main["e2e_enc_ms"] / 1e3), "unit": UNIT,
                 "h2d_bytes_per_step": main["h2d_enc"] * world, "d2h_bytes_per_step": 4 * world,
                 "call": "skipper_step_host_encoded: images + rates + labels H2D, on-device Poisson encoding, "
                         "step, loss D2H"} if "e2e_enc_ms" in main else
                {"value": gb * args.steps / (main["e2e_ms"] / 1e3), "unit": UNIT,
                 "h2d_bytes_per_step": main["h2d"] * world, "d2h_bytes_per_step": main["d2h"] * world,
                 "call": "skipper_step_host: spike frames + labels H2D, step, loss and s_t D2H"}),
        "e2e_spike_input": {"value": gb * args.steps / (main["e2e_ms"] / 1e3), "unit": UNIT,
                            "h2d_bytes_per_step": main["h2d"] * world, "d2h_bytes_per_step": main["d2h"] * world,
                            "call": "skipper_step_host: uint8 spike frames + labels H2D, step, loss D2H"},
        "gpu_launches": main["launches"],
        "clocks": main["clocks"],
        "kernels": breakdown,
        "step_roofline": {"roof_ms": roof_ms, "measured_ms": main["total_ms"] / args.steps,
                          "frac": roof_ms / (main["total_ms"] / args.steps),
                          "model": "sum over kernel classes of max(algorithmic FLOPs / sustained bf16 peak, "
                                   "algorithmic bytes / HBM peak), no overlap credit (SURVEY.md §8(d))"},
    }
    if world == 1 and not args.no_cpu_baseline:
        B_s = 2
        val, ms = oracle_samples_per_s(net, wl, args.mode, B_s, 1)
        line["cpu_baseline"] = {"value": val, "unit": UNIT, "cores": _CORES, "kind": "oracle",
                                "sample": f"1 step, B={B_s} of {wl['B']}, full T={wl['T']}, C={wl['C']}, p={wl['p']}, "
                                          f"mode={args.mode} ({ms / 1e3:.1f} s)"}
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="cfg2_vgg5")
    ap.add_argument("--mode", default="skip", choices=["skip", "ckpt", "full", "tbptt"])
    ap.add_argument("--T", type=int, default=0)
    ap.add_argument("--batch", type=int, default=0)
    ap.add_argument("--C", type=int, default=0)
    ap.add_argument("--p", type=float, default=None)
    ap.add_argument("--ref-batch", type=int, default=1)
    ap.add_argument("--group", type=int, default=1,
                    help="CKPT/SKIP backward groups (skipper_config.group): 1 = the paper's per-segment schedule")
    ap.add_argument("--no-compare", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--t-sweep", default="50,200,400", help="extra T values for peak-HBM / throughput vs T")
    ap.add_argument("--workloads", default="cfg3_vgg11,cfg4_resnet_dvs",
                    help="other BASELINE.json configs measured briefly in the same run (config.other_workloads)")
    ap.add_argument("--t-sweep-vgg11", default="100,500,1000,2000",
                    help="cfg 5: VGG-11 T values (B=128, C=5, p=50), all three modes; plus the C ~ sqrt(T) leg")
    ap.add_argument("--max-t", type=int, default=1, help="cfg 5: max-T search per mode (80 GB and device HBM)")
    args = ap.parse_args()
    if args.warmup < 3:
        raise SystemExit("--warmup must be >= 3")
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
