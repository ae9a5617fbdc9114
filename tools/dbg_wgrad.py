import sys, torch
sys.path.insert(0, '.')
from paper_conf_micro_singhslsknnd22_b200 import k_fc_wgrad, k_conv_wgrad
torch.backends.cuda.matmul.allow_tf32 = False
def bf(t): return t.to(torch.bfloat16).view(torch.int16).contiguous()
for (M, N, K) in [(640, 1024, 1024), (37, 24, 40), (1000, 136, 200)]:
    g = torch.Generator().manual_seed(M + K)
    D = torch.randint(-255, 256, (M, N), generator=g).float() * 2.0 ** -12
    X = (torch.rand((M, K), generator=g) < 0.3).float()
    ref = D.double().T @ X.double()
    Dd, Xd = bf(D).cuda(), bf(X).cuda()
    for it in range(4):
        out = k_fc_wgrad(Dd, Xd).cpu().double()
        e1 = (out - ref).abs().max().item()
        acc = torch.full((N, K), 0.5, device="cuda")
        torch.cuda.synchronize()
        k_fc_wgrad(Dd, Xd, out=acc)
        torch.cuda.synchronize()
        e2 = (acc.cpu().double() - 0.5 - ref).abs().max().item()
        acc2 = torch.zeros((N, K), device="cuda")
        k_fc_wgrad(Dd, Xd, out=acc2)
        e3 = (acc2.cpu().double() - ref).abs().max().item()
        print(M, N, K, it, "fresh", e1, "acc0.5", e2, "acc0", e3, "refmax", ref.abs().max().item(), flush=True)
