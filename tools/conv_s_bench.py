"""Micro-benchmark of the narrow / strided implicit conv (plan_conv_s) on the ResNet-DVS shapes:
achieved GB/s of (input once + fp32 output), optionally with SKIPPER_GEMM_STATS=1 pipeline waits."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_micro_singhslsknnd22_b200 import k_conv_s, k_fc_fwd


def bench(fn, it=10):
    for _ in range(2): fn()
    torch.cuda.synchronize()
    a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(it): fn()
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / it


def r(shape):
    return (torch.rand(shape, device="cuda") < 0.2).to(torch.bfloat16).view(torch.int16)


for (nb, h, w, cin, cout, s) in [(960, 64, 64, 16, 16, 1), (960, 32, 32, 16, 32, 2), (960, 32, 32, 32, 32, 1),
                                 (960, 16, 16, 32, 64, 2), (960, 16, 16, 64, 64, 1)]:
    X = r((nb, h * s, w * s, cin)); Wk = r((cout, 3, 3, cin))
    byt = X.numel() * 2 + nb * h * w * cout * 4
    for nw in (False, True):
        ms = bench(lambda: k_conv_s(X, Wk, stride=s, narrow=nw))
        print(f"conv_{'narrow' if nw else 's'} {nb}x{h}x{w} {cin}->{cout} s{s}: {ms*1e3:9.1f} us  {byt/ms/1e6:7.1f} GB/s",
              flush=True)
# the same work as an explicit-column GEMM (what the im2col path runs after staging)
M = 960 * 64 * 64
A = r((M, 144)); B = r((16, 144))
ms = bench(lambda: k_fc_fwd(A, B))
print(f"fc_fwd {M}x16x144: {ms*1e3:9.1f} us  {(A.numel()*2 + M*16*4)/ms/1e6:7.1f} GB/s")
