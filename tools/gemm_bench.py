"""Micro-benchmark of the tcgen05 GEMM kernels (warm, CUDA events): TF/s per shape."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_micro_singhslsknnd22_b200 import k_fc_fwd, k_conv_fwd, k_conv_dgrad, k_conv_wgrad, k_fc_wgrad

def bench(fn, flops, it=20):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(it): fn()
    b.record(); torch.cuda.synchronize()
    ms = a.elapsed_time(b) / it
    return ms, flops / ms / 1e9

def r(shape):
    return (torch.rand(shape, device="cuda") < 0.3).to(torch.bfloat16).view(torch.int16)

tag = os.environ.get("TAG", "")
for (nb, h, w, cin, cout) in [(640, 16, 16, 128, 128), (640, 16, 16, 64, 128), (160, 32, 32, 64, 64)]:
    X = r((nb, h, w, cin)); Wk = r((cout, 3, 3, cin))
    fl = 2.0 * nb * h * w * cout * 9 * cin
    ms, tf = bench(lambda: k_conv_fwd(X, Wk), fl)
    print(f"{tag} conv_fwd  {nb}x{h}x{w} {cin}->{cout}: {ms*1e3:8.1f} us  {tf:7.1f} TF/s")
    D = r((nb, h, w, cout)); Wt = r((cin, 3, 3, cout))
    ms, tf = bench(lambda: k_conv_dgrad(D, Wt), fl)
    print(f"{tag} conv_dgrad {nb}x{h}x{w} {cin}->{cout}: {ms*1e3:8.1f} us  {tf:7.1f} TF/s")
    out = torch.zeros((cout, 3, 3, cin), device="cuda")
    ms, tf = bench(lambda: k_conv_wgrad(D, X, out=out), fl)
    print(f"{tag} conv_wgrad {nb}x{h}x{w} {cin}->{cout}: {ms*1e3:8.1f} us  {tf:7.1f} TF/s")
for (M, N, K) in [(163840, 128, 1152), (163840, 256, 1024), (8192, 8192, 8192)]:
    A = r((M, K)); B = r((N, K))
    ms, tf = bench(lambda: k_fc_fwd(A, B), 2.0 * M * N * K)
    print(f"{tag} fc_fwd {M}x{N}x{K}: {ms*1e3:8.1f} us  {tf:7.1f} TF/s")
