"""Per-layer dW errors against the oracle with the fused dgrad + reverse scan on / off (same seeded inputs).

usage: python tools/fused_bwd_errs.py NAME T B [C p]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np
import torch

import synth
from oracle import StepConfig, train_step


def errs(g, r):
    g = np.asarray(g, np.float64)
    r = np.asarray(r, np.float64)
    return np.linalg.norm(g - r) / np.linalg.norm(r), np.abs(g - r).max() / np.abs(r).max()


def main():
    name, T, B = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
    C = int(sys.argv[4]) if len(sys.argv) > 4 else 2
    p = float(sys.argv[5]) if len(sys.argv) > 5 else 40.0
    from paper_conf_micro_singhslsknnd22_b200 import SkipperNet
    net = synth.net_config(name)
    W = synth.make_weights(net, seed=0)
    x, y = synth.make_inputs(net, T, B, seed=1)
    ref = train_step(net, W, x, y, StepConfig(T=T, C=C, p=p, mode="skip"))
    os.environ["SKIPPER_CL_MIN_UNITS"] = "0"
    dws = {}
    for fused in ("0", "1"):
        os.environ["SKIPPER_BWD_FUSION"] = fused
        m = SkipperNet(net, T, C=C, p=p, mode="skip", batch=B)
        m.set_weights(W)
        m.step(torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda())
        dws[fused] = [g.cpu().numpy() for g in m.grads()]
        m.close()
    for l, r in enumerate(ref.dW):
        e0, e1, ef = errs(dws["0"][l], r), errs(dws["1"][l], r), errs(dws["1"][l], dws["0"][l])
        print(f"{name} T={T} B={B} layer {l}: unfused {e0[0]:.2e}/{e0[1]:.2e}  fused {e1[0]:.2e}/{e1[1]:.2e}  "
              f"fused-vs-unfused {ef[0]:.2e}/{ef[1]:.2e}")


if __name__ == "__main__":
    main()
