"""Weight-gradient GEMM micro-benchmark (warm, CUDA events): conv wgrad (4D shifted boxes) vs fc wgrad
(2D boxes) on the same reduction sizes, VGG-11 / VGG-5 layer shapes."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_micro_singhslsknnd22_b200 import k_conv_wgrad, k_fc_wgrad

def bench(fn, flops, it=10):
    for _ in range(2): fn()
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
for (nb, h, w, cin, cout) in [(2560, 4, 4, 512, 512), (2560, 8, 8, 256, 256), (640, 16, 16, 128, 128), (640, 16, 16, 64, 128)]:
    X = r((nb, h, w, cin)); D = r((nb, h, w, cout))
    fl = 2.0 * nb * h * w * cout * 9 * cin
    out = torch.zeros((cout, 3, 3, cin), device="cuda")
    ms, tf = bench(lambda: k_conv_wgrad(D, X, out=out), fl)
    print(f"{tag} conv_wgrad {nb}x{h}x{w} {cin}->{cout}: {ms*1e3:8.1f} us  {tf:7.1f} TF/s", flush=True)
    M = nb * h * w
    Xc = r((M, 9 * cin)); Dm = D.view(M, cout)
    out2 = torch.zeros((cout, 9 * cin), device="cuda")
    ms, tf = bench(lambda: k_fc_wgrad(Dm, Xc, out=out2), fl)
    print(f"{tag} fc_wgrad   {M}x{cout}x{9*cin}: {ms*1e3:8.1f} us  {tf:7.1f} TF/s", flush=True)
