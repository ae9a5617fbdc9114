"""Time the fused conv + LIF kernel alone (CUDA events), optionally in a diagnostic mode.

usage: python tools/cl_bench.py [--R 10] [--nb 64] [--h 16] [--cin 128] [--cout 128] [--pool 1]
env: SKIPPER_CL_PAIR=0/1, SKIPPER_CL_DIAG=1 (no epilogue work) / 2 (no MMA) - results wrong when DIAG set
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

from paper_conf_micro_singhslsknnd22_b200 import k_conv_lif

ap = argparse.ArgumentParser()
ap.add_argument("--R", type=int, default=10)
ap.add_argument("--nb", type=int, default=64)
ap.add_argument("--h", type=int, default=16)
ap.add_argument("--cin", type=int, default=128)
ap.add_argument("--cout", type=int, default=128)
ap.add_argument("--pool", type=int, default=1)
ap.add_argument("--iters", type=int, default=20)
ap.add_argument("--store-u", type=int, default=0)
ap.add_argument("--graph", type=int, default=0, help="time a CUDA graph of --iters launches (no host launch cost)")
a = ap.parse_args()
X = (torch.rand(a.R, a.nb, a.h, a.h, a.cin, device="cuda") < 0.2).to(torch.bfloat16)
W = (torch.randint(-255, 256, (a.cout, 3, 3, a.cin), device="cuda").float() / 512).to(torch.bfloat16)
U = torch.zeros(a.nb, a.h, a.h, a.cout, device="cuda")
o = torch.zeros(a.nb, a.h, a.h, a.cout, dtype=torch.uint8, device="cuda")
for _ in range(3):
    k_conv_lif(X, W, U, o, a.pool, 0.99, 1.0, store_u=bool(a.store_u))
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
torch.cuda.synchronize()
if a.graph:
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(a.iters):
            k_conv_lif(X, W, U, o, a.pool, 0.99, 1.0, store_u=bool(a.store_u))
    g.replay()
    torch.cuda.synchronize()
e0.record()
if a.graph:
    g.replay()
else:
    for _ in range(a.iters):
        k_conv_lif(X, W, U, o, a.pool, 0.99, 1.0, store_u=bool(a.store_u))
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / a.iters
fl = 2.0 * a.R * a.nb * a.h * a.h * a.cout * 9 * a.cin
print(f"conv_lif R={a.R} nb={a.nb} {a.h}x{a.h} {a.cin}->{a.cout} pool={a.pool} pair={os.environ.get('SKIPPER_CL_PAIR', '1')} "
      f"diag={os.environ.get('SKIPPER_CL_DIAG', '0')} store_u={a.store_u}: {ms * 1e3:.1f} us  {fl / ms / 1e9:.0f} TF/s")
