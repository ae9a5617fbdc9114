"""Is the step launch-bound?  Host wall time per skipper_step (its one internal sync included) vs the
device time of the same steps (CUDA events).  usage: python tools/host_bound.py [--workload cfg2_vgg5]"""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_micro_singhslsknnd22_b200 import SkipperNet  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--workload", default="cfg2_vgg5")
ap.add_argument("--mode", default="skip")
ap.add_argument("--steps", type=int, default=20)
a = ap.parse_args()
wl = synth.workload(a.workload)
net = synth.net_config(wl["net"])
x, y = synth.make_inputs(net, wl["T"], wl["B"])
m = SkipperNet(net, wl["T"], C=wl["C"], p=wl["p"], mode=a.mode, batch=wl["B"])
m.set_weights(synth.make_weights(net))
xd, yd = torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda()
for _ in range(5):
    m.step(xd, yd, want_loss=False)
torch.cuda.synchronize()
st = torch.cuda.current_stream()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
host = []
e0.record(st)
for _ in range(a.steps):
    t0 = time.perf_counter()
    m.step(xd, yd, want_loss=False)
    host.append(time.perf_counter() - t0)
e1.record(st)
torch.cuda.synchronize()
dev = e0.elapsed_time(e1) / a.steps
print(f"{a.workload} {a.mode}: device {dev:.3f} ms/step, host call {1e3 * sum(host) / len(host):.3f} ms/step "
      f"(min {1e3 * min(host):.3f}), launches/step {m.launch_count() / (a.steps + 5):.0f}")
m.close()
