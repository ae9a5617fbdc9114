"""Run a few training steps of a workload (for ncu / compute-sanitizer; no timing)."""
import argparse, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
from paper_conf_micro_singhslsknnd22_b200 import SkipperNet

ap = argparse.ArgumentParser()
ap.add_argument("--workload", default="cfg2_vgg5")
ap.add_argument("--mode", default="skip")
ap.add_argument("--steps", type=int, default=2)
ap.add_argument("--batch", type=int, default=0)
ap.add_argument("--T", type=int, default=0)
a = ap.parse_args()
wl = synth.workload(a.workload)
if a.batch: wl["B"] = a.batch
if a.T: wl["T"] = a.T
net = synth.net_config(wl["net"])
x, y = synth.make_inputs(net, wl["T"], wl["B"])
m = SkipperNet(net, wl["T"], C=wl["C"], p=wl["p"], mode=a.mode, batch=wl["B"])
m.set_weights(synth.make_weights(net))
xd, yd = torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda()
for _ in range(a.steps):
    loss = m.step(xd, yd)
torch.cuda.synchronize()
print("loss", loss, "launches", m.launch_count())
