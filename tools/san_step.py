"""One small training step per network for compute-sanitizer (memcheck / racecheck / synccheck).
usage: python tools/san_step.py NAME T B C MODE"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_micro_singhslsknnd22_b200 import SkipperNet  # noqa: E402

name, T, B, C, mode = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4]), sys.argv[5]
net = synth.net_config(name)
x, y = synth.make_inputs(net, T, B)
m = SkipperNet(net, T, C=C, p=50.0 if mode == "skip" else 0.0, mode=mode, batch=B)
m.set_weights(synth.make_weights(net))
loss = m.step(torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda())
torch.cuda.synchronize()
print(f"{name} {mode} T={T} B={B} C={C}: loss {loss:.6f}, {m.launch_count()} launches")
m.close()
