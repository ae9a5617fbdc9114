import sys, torch
sys.path.insert(0, '.')
from paper_conf_micro_singhslsknnd22_b200 import k_fc_wgrad, lib
print("current stream", torch.cuda.current_stream(), torch.cuda.current_stream().cuda_stream)
def bf(t): return t.to(torch.bfloat16).view(torch.int16).contiguous()
M, N, K = 640, 1024, 1024
g = torch.Generator().manual_seed(M + K)
D = torch.randint(-255, 256, (M, N), generator=g).float() * 2.0 ** -12
X = (torch.rand((M, K), generator=g) < 0.3).float()
ref = D.double().T @ X.double()
for variant in ["as_test", "sync_before_cpu", "persistent_inputs", "as_test", "zeros_acc"]:
    out = k_fc_wgrad(bf(D).cuda(), bf(X).cuda()).cpu().double()
    e1 = (out - ref).abs().max().item()
    if variant == "zeros_acc":
        acc = torch.zeros((N, K), device="cuda")
        base = 0.0
    else:
        acc = torch.full((N, K), 0.5, device="cuda")
        base = 0.5
    if variant == "persistent_inputs":
        Dd, Xd = bf(D).cuda(), bf(X).cuda()
        k_fc_wgrad(Dd, Xd, out=acc)
    else:
        k_fc_wgrad(bf(D).cuda(), bf(X).cuda(), out=acc)
    if variant == "sync_before_cpu":
        torch.cuda.synchronize()
    got = acc.cpu().double()
    torch.cuda.synchronize()
    got2 = acc.cpu().double()
    e2 = (got - base - ref).abs().max().item()
    e3 = (got2 - base - ref).abs().max().item()
    print(variant, "fresh", e1, "acc", e2, "acc after sync", e3, flush=True)
