"""Per-layer weight-gradient error of the device step vs the oracle (diagnostic)."""
import sys
import numpy as np
import torch
sys.path.insert(0, ".")
import synth
from oracle import StepConfig, train_step
from paper_conf_micro_singhslsknnd22_b200 import SkipperNet

name, T, B, C, p, mode = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4]), float(sys.argv[5]), sys.argv[6]
net = synth.net_config(name)
W = synth.make_weights(net)
x, y = synth.make_inputs(net, T, B)
for emu in (True, False):
    ref = train_step(net, W, x, y, StepConfig(T=T, C=C, p=p, mode=mode, emulate_bf16=emu))
    m = SkipperNet(net, T, C=C, p=p, mode=mode, batch=B)
    m.set_weights(W)
    m.step(torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda())
    errs = []
    for l, (g, r) in enumerate(zip(m.grads(), ref.dW)):
        g = g.cpu().numpy().astype(np.float64)
        errs.append(np.linalg.norm(g - r) / max(np.linalg.norm(r), 1e-300))
    print("emulate_bf16", emu, " ".join(f"{e:.1e}" for e in errs))
    m.close()
