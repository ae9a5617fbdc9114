import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_micro_singhslsknnd22_b200 import k_conv_s
X = (torch.rand((960, 64, 64, 16), device="cuda") < 0.2).to(torch.bfloat16).view(torch.int16)
W = (torch.rand((16, 3, 3, 16), device="cuda") < 0.2).to(torch.bfloat16).view(torch.int16)
for _ in range(2):
    k_conv_s(X, W, narrow=True)
torch.cuda.synchronize()
