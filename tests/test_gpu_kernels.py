"""Per-kernel parity of the tcgen05/TMA synaptic contractions (K2) against a plain
PyTorch float64 reference of the same op.  Inputs are exact in bf16; spike-like
operands with grid weights make every fp32 sum exact, so those cases must match
bit for bit; random-normal cases are checked to fp32-accumulation tolerance."""
import pytest
import torch
import torch.nn.functional as F

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_micro_singhslsknnd22_b200 as pk  # noqa: F401  (fails loudly if the .so is missing)
    torch.backends.cuda.matmul.allow_tf32 = False
    torch.backends.cudnn.allow_tf32 = False


def bf16_bits(t):
    return t.to(torch.bfloat16).view(torch.int16).contiguous()


def spikes(shape, rate=0.3, gen=None):
    return (torch.rand(shape, generator=gen) < rate).float()


def grid(shape, e=8, gen=None):
    return torch.randint(-255, 256, shape, generator=gen).float() * 2.0 ** -e


@pytest.mark.parametrize("M,N,K", [(640, 1024, 8192), (100, 128, 784), (37, 24, 40), (300, 264, 136),
                                   (1, 8, 8), (257, 512, 1024), (129, 64, 64)])
def test_fc_fwd_exact(M, N, K):
    from paper_conf_micro_singhslsknnd22_b200 import k_fc_fwd
    g = torch.Generator().manual_seed(M * 7 + N)
    A = spikes((M, K), gen=g)
    B = grid((N, K), gen=g)
    ref = (A.double() @ B.double().T).float()
    out = k_fc_fwd(bf16_bits(A).cuda(), bf16_bits(B).cuda()).cpu()
    assert torch.equal(out, ref), (out - ref).abs().max()


def test_fc_fwd_random_normal():
    from paper_conf_micro_singhslsknnd22_b200 import k_fc_fwd
    g = torch.Generator().manual_seed(0)
    A = torch.randn(333, 704, generator=g).bfloat16()
    B = torch.randn(200, 704, generator=g).bfloat16()
    ref = A.double() @ B.double().T
    out = k_fc_fwd(A.view(torch.int16).cuda(), B.view(torch.int16).cuda()).cpu().double()
    assert (out - ref).norm() / ref.norm() < 1e-6


@pytest.mark.parametrize("M,N,K", [(640, 1024, 1024), (80, 128, 784), (37, 24, 40), (1000, 136, 200),
                                   (4096, 64, 128)])
def test_fc_wgrad(M, N, K):
    from paper_conf_micro_singhslsknnd22_b200 import k_fc_wgrad
    g = torch.Generator().manual_seed(M + K)
    D = grid((M, N), e=12, gen=g)
    X = spikes((M, K), gen=g)
    ref = D.double().T @ X.double()
    out = k_fc_wgrad(bf16_bits(D).cuda(), bf16_bits(X).cuda()).cpu().double()
    assert (out - ref).abs().max() <= 1e-6 * ref.abs().max() + 1e-12
    # accumulate mode adds into the existing buffer
    acc = torch.full((N, K), 0.5, dtype=torch.float32, device="cuda")
    k_fc_wgrad(bf16_bits(D).cuda(), bf16_bits(X).cuda(), out=acc)
    assert (acc.cpu().double() - 0.5 - ref).abs().max() <= 1e-6 * ref.abs().max() + 1e-6


CONV_SHAPES = [(6, 16, 16, 64, 128), (3, 8, 8, 128, 256), (5, 4, 4, 64, 64), (33, 2, 2, 64, 128),
               (2, 32, 32, 64, 64), (7, 16, 16, 128, 128), (3, 4, 4, 512, 512)]


def conv_ref(X, W):  # X [nb][h][w][ci], W [co][3][3][ci]
    return F.conv2d(X.permute(0, 3, 1, 2).double(), W.permute(0, 3, 1, 2).double(), padding=1).permute(0, 2, 3, 1)


@pytest.mark.parametrize("nb,h,w,cin,cout", CONV_SHAPES)
def test_conv_fwd_exact(nb, h, w, cin, cout):
    from paper_conf_micro_singhslsknnd22_b200 import k_conv_fwd
    g = torch.Generator().manual_seed(nb * h + cin)
    X = spikes((nb, h, w, cin), gen=g) * 0.25 * torch.randint(0, 5, (nb, h, w, cin), generator=g)  # pooled values
    W = grid((cout, 3, 3, cin), gen=g)
    ref = conv_ref(X, W).float()
    out = k_conv_fwd(bf16_bits(X).cuda(), bf16_bits(W).cuda()).cpu()
    assert torch.equal(out, ref), (out - ref).abs().max()


@pytest.mark.parametrize("nb,h,w,cin,cout", CONV_SHAPES)
def test_conv_dgrad(nb, h, w, cin, cout):
    from paper_conf_micro_singhslsknnd22_b200 import k_conv_dgrad
    g = torch.Generator().manual_seed(nb * w + cout)
    D = grid((nb, h, w, cout), e=10, gen=g)
    W = grid((cout, 3, 3, cin), gen=g)
    X = torch.zeros((nb, h, w, cin), dtype=torch.float64, requires_grad=True)
    conv_ref(X, W).backward(D.double())
    ref = X.grad
    Wt = W.permute(3, 1, 2, 0).contiguous()  # [cin][3][3][cout]
    out = k_conv_dgrad(bf16_bits(D).cuda(), bf16_bits(Wt).cuda()).cpu().double()
    assert (out - ref).abs().max() <= 1e-6 * ref.abs().max() + 1e-12


@pytest.mark.parametrize("nb,h,w,cin,cout", CONV_SHAPES)
def test_conv_wgrad(nb, h, w, cin, cout):
    from paper_conf_micro_singhslsknnd22_b200 import k_conv_wgrad
    g = torch.Generator().manual_seed(nb + h + cout)
    D = grid((nb, h, w, cout), e=12, gen=g)
    X = spikes((nb, h, w, cin), gen=g)
    Wv = torch.zeros((cout, 3, 3, cin), dtype=torch.float64, requires_grad=True)
    conv_ref(X, Wv).backward(D.double())
    ref = Wv.grad
    out = k_conv_wgrad(bf16_bits(D).cuda(), bf16_bits(X).cuda()).cpu().double()
    assert (out - ref).abs().max() <= 1e-5 * ref.abs().max() + 1e-12


NARROW_WGRAD_SHAPES = [(3, 64, 64, 16, 16, 1), (2, 32, 32, 32, 32, 1), (5, 16, 16, 16, 32, 1), (3, 32, 32, 16, 32, 2),
                       (2, 16, 16, 32, 64, 2), (4, 16, 16, 32, 16, 1), (7, 4, 16, 16, 64, 1)]


@pytest.mark.parametrize("nb,h,w,cin,cout,stride", NARROW_WGRAD_SHAPES)
def test_narrow_wgrad(nb, h, w, cin, cout, stride):
    """Narrow-channel weight gradient (ldmatrix row gathers, no column buffer) against the float64 conv
    backward, for stride 1 and 2 and every (cin, cout) the ResNet layers use; h x w is the output size."""
    from paper_conf_micro_singhslsknnd22_b200 import k_narrow_wgrad
    g = torch.Generator().manual_seed(nb * 7 + h + cout + stride)
    D = grid((nb, h, w, cout), e=12, gen=g)
    X = spikes((nb, stride * h, stride * w, cin), gen=g)
    Wv = torch.zeros((cout, 3, 3, cin), dtype=torch.float64, requires_grad=True)
    y = F.conv2d(X.permute(0, 3, 1, 2).double(), Wv.permute(0, 3, 1, 2), padding=1, stride=stride).permute(0, 2, 3, 1)
    y.backward(D.double())
    ref = Wv.grad
    out = k_narrow_wgrad(bf16_bits(D).cuda(), bf16_bits(X).cuda(), stride=stride).cpu().double()
    assert (out - ref).abs().max() <= 1e-5 * ref.abs().max() + 1e-12
    acc = out.float().cuda()
    k_narrow_wgrad(bf16_bits(D).cuda(), bf16_bits(X).cuda(), stride=stride, out=acc)  # accumulates
    assert (acc.cpu().double() - 2 * ref).abs().max() <= 2e-5 * ref.abs().max() + 1e-12


@pytest.mark.parametrize("nb,h,w,cin,cout,stride", [(3, 64, 64, 16, 16, 1), (2, 32, 32, 32, 32, 1), (5, 16, 16, 16, 32, 1),
                                                     (4, 16, 16, 32, 16, 1), (7, 4, 16, 16, 16, 1), (2, 8, 32, 32, 32, 1),
                                                     (3, 32, 32, 16, 32, 2), (2, 16, 16, 32, 64, 2), (5, 8, 8, 16, 16, 2)])
def test_narrow_dgrad(nb, h, w, cin, cout, stride):
    """Narrow dgrad (staged delta rows, ldmatrix gathers; stride 1 and 2) against the float64 conv input
    gradient; h x w is the output size.  Spike-like delta and grid weights make every fp32 sum exact."""
    from paper_conf_micro_singhslsknnd22_b200 import k_narrow_dgrad
    g = torch.Generator().manual_seed(nb * 11 + h + cin + cout + stride)
    W = grid((cout, 3, 3, cin), gen=g)
    D = spikes((nb, h, w, cout), gen=g)
    X = torch.zeros((nb, stride * h, stride * w, cin), dtype=torch.float64, requires_grad=True)
    y = F.conv2d(X.permute(0, 3, 1, 2), W.permute(0, 3, 1, 2).double(), padding=1, stride=stride).permute(0, 2, 3, 1)
    y.backward(D.double())
    ref = X.grad
    Wt = W.permute(3, 1, 2, 0).contiguous()  # [cin][3][3][cout]
    out = k_narrow_dgrad(bf16_bits(D).cuda(), bf16_bits(Wt).cuda(), stride=stride).cpu().double()
    assert torch.equal(out, ref)


def test_stream_ordering_with_torch():
    """The library's kernels are ordered with torch's work on the same stream: a long GEMM
    followed immediately by a torch copy of its output must see the finished result."""
    from paper_conf_micro_singhslsknnd22_b200 import k_fc_fwd
    M, N, K = 1 << 16, 1024, 4096
    A = torch.ones((M, K), dtype=torch.bfloat16, device="cuda")
    B = torch.full((N, K), 0.5, dtype=torch.bfloat16, device="cuda")
    for _ in range(3):
        out = k_fc_fwd(A.view(torch.int16), B.view(torch.int16))
        host = out.cpu()                      # no explicit synchronize
        assert torch.all(host == K * 0.5)
        side = torch.cuda.Stream()
        with torch.cuda.stream(side):
            out2 = k_fc_fwd(A.view(torch.int16), B.view(torch.int16))
            h2 = out2.cpu()
        assert torch.all(h2 == K * 0.5)


CONV_LIF_SHAPES = [(5, 6, 16, 16, 64, 128, 1), (4, 3, 8, 8, 128, 256, 0), (3, 5, 4, 4, 64, 64, 1),
                   (6, 2, 32, 32, 64, 64, 1), (3, 7, 16, 16, 128, 128, 0), (1, 2, 16, 16, 64, 128, 1)]


@pytest.mark.parametrize("variant", ["single", "single_tap_boxes", "pair", "pair_streamed_w"])
@pytest.mark.parametrize("R,nb,h,w,cin,cout,pool", CONV_LIF_SHAPES)
def test_conv_lif_exact(R, nb, h, w, cin, cout, pool, variant, monkeypatch):
    """Fused conv + LIF (Eq.1) against conv2d in float64 (exact on the grid, rounded once to fp32) and
    the LIF update in fp32 without FMA; spikes, pooled outputs and final state bit-exact."""
    from paper_conf_micro_singhslsknnd22_b200 import k_conv_lif
    monkeypatch.setenv("SKIPPER_CL_PAIR", "0" if variant == "single" else "1")  # CTA pair (cta_group::2)
    monkeypatch.setenv("SKIPPER_CL_RESB", "0" if variant == "pair_streamed_w" else "1")  # resident weights
    monkeypatch.setenv("SKIPPER_CL_HALO", "0" if variant == "single_tap_boxes" else "1")  # halo activation boxes
    g = torch.Generator().manual_seed(R * 131 + nb * h + cin + pool)
    X = spikes((R, nb, h, w, cin), gen=g) * 0.25 * torch.randint(1, 5, (R, nb, h, w, cin), generator=g)
    W = grid((cout, 3, 3, cin), e=9, gen=g)
    U0 = grid((nb, h, w, cout), e=9, gen=g) * 0.5
    o0 = (torch.rand((nb, h, w, cout), generator=g) < 0.2).to(torch.uint8)
    lam, theta = 0.75, 1.0
    U, o = U0.clone(), o0.float()
    refP, refU = [], []
    for r in range(R):
        I = conv_ref(X[r], W).float()
        U = (lam * U + I) - theta * o
        o = (U > theta).float()
        refU.append(U.clone())
        refP.append(F.avg_pool2d(o.permute(0, 3, 1, 2), 2).permute(0, 2, 3, 1) if pool else o.clone())
    Us, os_ = U0.clone().cuda(), o0.clone().cuda()
    P, Uo = k_conv_lif(bf16_bits(X).cuda(), bf16_bits(W).cuda(), Us, os_, pool, lam, theta)
    P = P.cpu().float()
    for r in range(R):
        assert torch.equal(P[r], refP[r]), f"row {r}: {int((P[r] != refP[r]).sum())} outputs differ"
        assert torch.equal(Uo[r].cpu(), refU[r]), f"row {r}: U max diff {(Uo[r].cpu() - refU[r]).abs().max()}"
    assert torch.equal(Us.cpu(), refU[-1])
    assert torch.equal(os_.cpu(), (refU[-1] > theta).to(torch.uint8))


CONV_S_SHAPES = [  # nb, output h, w, cin, cout, stride  (ResNet-DVS layers and ragged / multi-image tiles)
    (3, 64, 64, 16, 16, 1), (2, 32, 32, 16, 32, 2), (2, 32, 32, 32, 32, 1), (2, 16, 16, 32, 64, 2),
    (3, 8, 8, 16, 16, 1), (5, 4, 4, 16, 32, 2), (3, 16, 16, 64, 64, 2), (2, 8, 8, 32, 16, 1)]


@pytest.mark.parametrize("narrow", [False, True])
@pytest.mark.parametrize("nb,h,w,cin,cout,stride", CONV_S_SHAPES)
def test_conv_s_exact(nb, h, w, cin, cout, stride, narrow):
    """Narrow-channel / strided implicit conv (per-tap 32B/64B-swizzled TMA boxes, TMA element strides)
    against torch conv2d(stride, padding=1) in float64: exact for spikes x grid weights."""
    from paper_conf_micro_singhslsknnd22_b200 import k_conv_s
    g = torch.Generator().manual_seed(nb * 131 + h + cin + stride)
    X = spikes((nb, h * stride, w * stride, cin), gen=g)
    W = grid((cout, 3, 3, cin), gen=g)
    ref = F.conv2d(X.permute(0, 3, 1, 2).double(), W.permute(0, 3, 1, 2).double(), padding=1,
                   stride=stride).permute(0, 2, 3, 1).float()
    out = k_conv_s(bf16_bits(X).cuda(), bf16_bits(W).cuda(), stride=stride, narrow=narrow).cpu()
    assert torch.equal(out, ref), (out - ref).abs().max()


@pytest.mark.parametrize("narrow", [False, True])
@pytest.mark.parametrize("nb,h,w,cin,cout", [(3, 64, 64, 16, 16), (2, 32, 32, 32, 32), (2, 8, 8, 32, 16),
                                             (2, 16, 16, 64, 64)])
def test_conv_s_dgrad_exact(nb, h, w, cin, cout, narrow):
    """Stride-1 dgrad through the narrow path: G = conv_transpose(D, W) = conv(D, flipped W^T)."""
    from paper_conf_micro_singhslsknnd22_b200 import k_conv_s
    g = torch.Generator().manual_seed(nb + h + cin)
    D = grid((nb, h, w, cout), e=10, gen=g)
    W = grid((cout, 3, 3, cin), gen=g)
    ref = F.conv_transpose2d(D.permute(0, 3, 1, 2).double(), W.permute(0, 3, 1, 2).double(),
                             padding=1).permute(0, 2, 3, 1).float()
    Wt = W.permute(3, 1, 2, 0).contiguous()          # [cin][3][3][cout]
    out = k_conv_s(bf16_bits(D).cuda(), bf16_bits(Wt).cuda(), stride=1, sign=-1, narrow=narrow).cpu()
    assert torch.equal(out, ref), (out - ref).abs().max()
