"""Per-phase device time of one training step (profile mode: every launch bracketed by CUDA events, the weight
gradients serialised on the main stream): first-pass forward, recompute forward, backward, optimizer - the
measured F and B of DESIGN.md §8's Skipper-vs-BPTT condition B / F > k / (1 - k).

usage: python tools/phase_split.py [--workload cfg2_vgg5] [--steps 3]"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_micro_singhslsknnd22_b200 import SkipperNet  # noqa: E402

FWD = {"stage_input", "gemm_fwd", "lif_fwd_scan", "layer0_fused_fwd", "gemm_lif_fwd", "im2col_fwd"}
OPT = {"adam"}


def split(workload, mode, steps):
    wl = synth.workload(workload)
    net = synth.net_config(wl["net"])
    x, y = synth.make_inputs(net, wl["T"], wl["B"])
    m = SkipperNet(net, wl["T"], C=wl["C"], p=wl["p"], mode=mode, batch=wl["B"])
    m.set_weights(synth.make_weights(net))
    xd, yd = torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda()
    for _ in range(3):
        m.step(xd, yd, want_loss=False)
    torch.cuda.synchronize()
    m.profile(True)
    for _ in range(steps):
        m.step(xd, yd, want_loss=False)
    recs = m.profile_records()
    m.profile(False)
    m.close()
    n = len(recs) // steps
    out = {"first": 0.0, "recompute": 0.0, "backward": 0.0, "optimizer": 0.0}
    for s in range(steps):
        seen_loss = False
        for c, k, by, fl, ms in recs[s * n:(s + 1) * n]:
            if c == "readout_loss" and not seen_loss:   # finish_first: the loss ends the first pass
                seen_loss = True
                out["first" if mode != "full" else "first"] += ms
                continue
            if c in OPT:
                out["optimizer"] += ms
            elif c in FWD:
                out["recompute" if seen_loss else "first"] += ms
            else:
                out["backward"] += ms
    return {k: round(v / steps, 3) for k, v in out.items()}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="cfg2_vgg5")
    ap.add_argument("--steps", type=int, default=3)
    a = ap.parse_args()
    res = {mode: split(a.workload, mode, a.steps) for mode in ("full", "skip")}
    full, skip = res["full"], res["skip"]
    F, B = full["first"], full["backward"]
    res["B_over_F_full"] = round(B / F, 3)
    res["workload"] = a.workload
    print(json.dumps(res))


if __name__ == "__main__":
    main()
