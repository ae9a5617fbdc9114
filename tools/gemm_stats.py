"""One launch per GEMM shape with SKIPPER_GEMM_STATS=1 (barrier wait fractions per role)."""
import os, sys
os.environ["SKIPPER_GEMM_STATS"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_micro_singhslsknnd22_b200 import k_fc_fwd, k_conv_fwd, k_conv_dgrad, k_conv_wgrad, k_fc_wgrad
def r(shape):
    return (torch.rand(shape, device="cuda") < 0.3).to(torch.bfloat16).view(torch.int16)
for (nb, h, w, cin, cout) in [(640, 16, 16, 128, 128), (640, 16, 16, 64, 128)]:
    X = r((nb, h, w, cin)); Wk = r((cout, 3, 3, cin)); D = r((nb, h, w, cout)); Wt = r((cin, 3, 3, cout))
    for _ in range(2):
        k_conv_fwd(X, Wk); k_conv_dgrad(D, Wt); k_conv_wgrad(D, X)
for (M, N, K) in [(8192, 8192, 8192), (163840, 256, 1024), (640, 1024, 8192)]:
    A = r((M, K)); B = r((N, K))
    for _ in range(2):
        k_fc_fwd(A, B)
D = r((640, 1024)); X = r((640, 8192))
k_fc_wgrad(D, X); k_fc_wgrad(D, X)
torch.cuda.synchronize()
