import sys, torch
sys.path.insert(0, '.')
from paper_conf_micro_singhslsknnd22_b200 import k_fc_wgrad, k_fc_fwd
def bf(t): return t.to(torch.bfloat16).view(torch.int16).contiguous()
def wg(M, N, K, tag):
    g = torch.Generator().manual_seed(M + K)
    D = torch.randint(-255, 256, (M, N), generator=g).float() * 2.0 ** -12
    X = (torch.rand((M, K), generator=g) < 0.3).float()
    ref = D.double().T @ X.double()
    out = k_fc_wgrad(bf(D).cuda(), bf(X).cuda()).cpu().double()
    e1 = (out - ref).abs().max().item()
    acc = torch.full((N, K), 0.5, device="cuda")
    k_fc_wgrad(bf(D).cuda(), bf(X).cuda(), out=acc)
    e2 = (acc.cpu().double() - 0.5 - ref).abs().max().item()
    print(tag, M, N, K, "fresh", e1, "acc", e2, flush=True)
wg(640, 1024, 1024, "cold")
for (M, N, K) in [(640, 1024, 8192), (100, 128, 784), (37, 24, 40), (300, 264, 136), (1, 8, 8), (257, 512, 1024), (129, 64, 64)]:
    g = torch.Generator().manual_seed(M * 7 + N)
    A = (torch.rand((M, K), generator=g) < 0.3).float()
    B = torch.randint(-255, 256, (N, K), generator=g).float() * 2.0 ** -8
    ref = (A.double() @ B.double().T).float()
    out = k_fc_fwd(bf(A).cuda(), bf(B).cuda()).cpu()
    print("fwd", M, N, K, torch.equal(out, ref))
wg(640, 1024, 1024, "after-fwd")
wg(640, 1024, 1024, "again")
wg(80, 128, 784, "again")
