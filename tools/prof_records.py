"""Per-launch CUDA-event times of one training step in profile mode (serialised wgrad), grouped in order.
usage: python tools/prof_records.py [--workload cfg2_vgg5] [--mode skip] [--steps 3]"""
import argparse
import collections
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_micro_singhslsknnd22_b200 import SkipperNet  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--workload", default="cfg2_vgg5")
ap.add_argument("--mode", default="skip")
ap.add_argument("--steps", type=int, default=3)
ap.add_argument("--all", action="store_true")
a = ap.parse_args()
wl = synth.workload(a.workload)
net = synth.net_config(wl["net"])
x, y = synth.make_inputs(net, wl["T"], wl["B"])
m = SkipperNet(net, wl["T"], C=wl["C"], p=wl["p"], mode=a.mode, batch=wl["B"])
m.set_weights(synth.make_weights(net))
xd, yd = torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda()
for _ in range(3):
    m.step(xd, yd, want_loss=False)
torch.cuda.synchronize()
m.profile(True)
for _ in range(a.steps):
    m.step(xd, yd, want_loss=False)
recs = m.profile_records()
m.profile(False)
n = len(recs) // a.steps
recs = recs[-n:]
tot = collections.defaultdict(float)
for i, (c, k, by, fl, ms) in enumerate(recs):
    tot[c] += ms
    if a.all:
        print(f"{i:4d} {c:18s} {ms * 1e3:8.1f} us  {by / 1e6:8.2f} MB  {fl / 1e9:8.2f} GF  "
              f"{by / max(ms, 1e-9) / 1e6:7.0f} GB/s {fl / max(ms, 1e-9) / 1e9:6.0f} TF/s")
print({k: round(v, 3) for k, v in sorted(tot.items(), key=lambda kv: -kv[1])}, "sum", round(sum(tot.values()), 3))
