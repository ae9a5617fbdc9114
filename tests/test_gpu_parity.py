"""End-to-end parity of the CUDA training step (through the C ABI) with the CPU
oracle on the same seeded inputs (SURVEY.md §8(c) tolerances):
  spikes bit-exact (first pass and recompute), membranes within 1e-5 relative
  (bit-exact expected under the arithmetic contract), s_t and keep masks exact,
  weight gradients within 1e-3 (normwise and max-abs), loss within 1e-5,
  post-Adam weights where the gradient is significant."""
import numpy as np
import pytest
import torch

import synth
from oracle import StepConfig, adam_update, train_step

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"


def run_gpu(net, W, x, y, T, C, p, mode, steps=1, sam="spikes", surrogate="triangle", gamma=0.3, group=1):
    from paper_conf_micro_singhslsknnd22_b200 import SkipperNet
    B = x.shape[1]
    m = SkipperNet(net, T, C=C, p=p, mode=mode, batch=B, debug_record=True, sam=sam, surrogate=surrogate,
                   gamma=gamma, group=group)
    m.set_weights(W)
    xd = torch.from_numpy(np.ascontiguousarray(x)).cuda()
    yd = torch.from_numpy(np.ascontiguousarray(y)).cuda()
    loss = m.step(xd, yd)
    return m, loss


def grad_errs(g, r):
    """(normwise, max-abs) relative error of g against r."""
    g = np.asarray(g, np.float64)
    r = np.asarray(r, np.float64)
    return np.linalg.norm(g - r) / np.linalg.norm(r), np.abs(g - r).max() / np.abs(r).max()


def grad_ok(g, r, tol=(1e-3, 1e-3)):
    g = np.asarray(g, np.float64)
    r = np.asarray(r, np.float64)
    if np.linalg.norm(r) == 0:
        return np.abs(g).max() == 0, "zero ref"
    rel, mx = grad_errs(g, r)
    return rel <= tol[0] and mx <= tol[1], f"normwise {rel:.2e} maxabs {mx:.2e}"


def check_parity(name, T, B, C, p, mode, lam=None, seed=0, sam="spikes", deep=False, theta=None, wscale=1.0,
                 surrogate="triangle", gamma=0.3, x_fn=None, group=1):
    """deep=True (networks deeper than the 11 spiking layers of VGG-11): a layer's dW tolerance is
    max(1e-3, twice the size of the bf16 contract's own effect on that layer), normwise and max-abs,
    DESIGN.md §4 "deep networks".  theta / wscale: threshold of every spiking layer and a power-of-two
    scale of their (grid) weights; surrogate / gamma: reading 4; x_fn: transforms the seeded input."""
    net = synth.net_config(name, lam=lam, theta=theta)
    W = synth.make_weights(net, seed=seed)
    W = [w * np.float32(wscale) if L["kind"] != "readout" else w for w, L in zip(W, net["layers"])]
    x, y = synth.make_inputs(net, T, B, seed=seed + 1)
    if x_fn is not None:
        x = np.ascontiguousarray(x_fn(x))
    ref = train_step(net, W, x, y, StepConfig(T=T, C=C, p=p, mode=mode, record=True, sam=sam, surrogate=surrogate,
                                              gamma=gamma))
    tols = [(1e-3, 1e-3)] * len(ref.dW)
    if deep:
        exact = train_step(net, W, x, y, StepConfig(T=T, C=C, p=p, mode=mode, sam=sam, emulate_bf16=False,
                                                     surrogate=surrogate, gamma=gamma))
        tols = []
        for a, b in zip(ref.dW, exact.dW):
            en, em = grad_errs(b, a)
            tols.append((max(1e-3, 2 * en), max(1e-3, 2 * em)))
    m, loss = run_gpu(net, W, x, y, T, C, p, mode, sam=sam, surrogate=surrogate, gamma=gamma, group=group)
    spk = [L for L in net["layers"] if L["kind"] != "readout"]
    # SAM and mask (Eq.4, Eq.5)
    np.testing.assert_array_equal(m.spike_sums(), ref.s)
    np.testing.assert_array_equal(m.layer_spike_counts(), ref.counts)
    if sam == "l2trace":  # float64 sums of exact squares: only the summation order differs
        np.testing.assert_allclose(m.sam_values(), np.asarray(ref.sam, np.float64), rtol=1e-12)
    else:
        np.testing.assert_array_equal(m.sam_values(), np.asarray(ref.sam, np.float64))  # same fp64 arithmetic
    np.testing.assert_array_equal(m.keep_mask(), ref.keep)
    # first pass and recomputed states per layer
    for l in range(len(spk)):
        fo = m.debug(1, l).cpu().numpy()
        assert np.array_equal(fo, ref.first_o[l]), f"layer {l}: {np.count_nonzero(fo != ref.first_o[l])} first-pass spikes differ"
        fU = m.debug(0, l).cpu().numpy()
        np.testing.assert_allclose(fU, ref.first_U[l], rtol=1e-5, atol=1e-6)
        ro = m.debug(3, l).cpu().numpy()
        assert np.array_equal(ro, ref.rec_o[l]), f"layer {l}: {np.count_nonzero(ro != ref.rec_o[l])} recomputed spikes differ"
        rU = m.debug(2, l).cpu().numpy()
        np.testing.assert_allclose(rU, ref.rec_U[l], rtol=1e-5, atol=1e-6)
    assert loss == pytest.approx(ref.loss, rel=1e-5)
    grads = m.grads()
    for l, (g, r) in enumerate(zip(grads, ref.dW)):
        ok, msg = grad_ok(g.cpu().numpy(), r, tols[l])
        assert ok, f"layer {l} dW: {msg} (tolerance {tols[l][0]:.1e}, {tols[l][1]:.1e})"
    # one Adam step from the shared starting point
    w_new = m.weights()
    for l, (wn, w0, r, g) in enumerate(zip(w_new, W, ref.dW, grads)):
        wn = wn.cpu().numpy().astype(np.float64)
        g = g.cpu().numpy().astype(np.float64)
        # (a) the optimizer kernel itself: fp64 Adam applied to the gradient the device produced
        wg, _, _ = adam_update(w0, g, np.zeros_like(g), np.zeros_like(g), 1)
        np.testing.assert_allclose(wn, wg, rtol=1e-6, atol=1e-8)
        # (b) end to end against the oracle where the first step is well conditioned: the update
        # g / (|g| + eps) amplifies a relative gradient error by eps/|g|, so compare where |g| is well
        # above eps, outside the cancelling tail, and the gradient element agrees to 1%
        sig = (np.abs(r) > max(1e-3 * np.abs(r).max(), 1e-6)) & (np.abs(g - r) <= 1e-2 * np.abs(r))
        wr, _, _ = adam_update(w0, r, np.zeros_like(r), np.zeros_like(r), 1)
        np.testing.assert_allclose(wn[sig], wr[sig], rtol=0, atol=2e-6)
    return m, ref


@pytest.mark.parametrize("mode", ["full", "ckpt", "skip"])
def test_cfg1_fc784_full_size(mode):
    """BASELINE.json configs[0]: 784-128-10, T=20, B=4, C=2, p=50."""
    check_parity("fc784", T=20, B=4, C=2, p=50.0, mode=mode)


@pytest.mark.parametrize("mode,lam", [("full", 1.0), ("ckpt", 0.99), ("skip", 0.5), ("skip", 0.99)])
def test_tiny_fc(mode, lam):
    check_parity("tiny_fc", T=12, B=3, C=2, p=40.0, mode=mode, lam=lam)


@pytest.mark.parametrize("mode,lam", [("full", 0.99), ("ckpt", 1.0), ("skip", 0.99), ("skip", 0.75)])
def test_tiny_conv(mode, lam):
    check_parity("tiny_conv", T=12, B=3, C=2, p=50.0, mode=mode, lam=lam)


@pytest.mark.parametrize("name,T,B,theta,wscale,surrogate,gamma", [
    ("tiny_conv", 12, 3, 2.0, 2.0, "triangle", 0.3), ("tiny_conv", 12, 3, 0.5, 1.0, "triangle", 0.3),
    ("tiny_fc", 12, 3, 0.5, 0.5, "fast_sigmoid", 2.0), ("tiny_conv", 12, 3, 1.0, 1.0, "fast_sigmoid", 4.0),
    ("vgg5", 14, 2, 2.0, 2.0, "fast_sigmoid", 1.0), ("tiny_resnet", 16, 3, 0.5, 0.5, "triangle", 0.5),
    ("fc784", 20, 4, 2.0, 2.0, "triangle", 0.3)])
def test_theta_and_surrogate(name, T, B, theta, wscale, surrogate, gamma):
    """theta != 1 (the /theta of the triangle surrogate and the theta*o reset, reading 1 and 4) and the
    fast-sigmoid surrogate (reading 4) on the device, every kernel kind that evaluates sigma'."""
    check_parity(name, T=T, B=B, C=2, p=50.0, mode="skip", theta=theta, wscale=wscale, surrogate=surrogate,
                 gamma=gamma)


@pytest.mark.parametrize("name,T,B,C,p,pulse", [("tiny_conv", 12, 3, 2, 90.0, True), ("tiny_conv", 12, 3, 2, 99.0, False),
                                                ("vgg5", 24, 2, 2, 95.0, True), ("tiny_fc", 12, 3, 2, 99.0, True),
                                                ("tiny_resnet", 16, 2, 2, 99.0, True), ("fc784", 20, 4, 2, 99.0, True)])
def test_high_p_single_row_segments(name, T, B, C, p, pulse):
    """p above the Eq.7 rule of thumb (accepted with a warning, reading 20).  pulse: the input fires only at the
    segment starts t = cS, so s_{cS} is each segment's maximum and every other step falls below SST_c: the
    segments shrink to K_c = 1 (only the checkpoint row is recomputed and back-propagated)."""
    S = T // C
    fn = (lambda x: np.where((np.arange(x.shape[0]) % S == 0).reshape((-1,) + (1,) * (x.ndim - 1)), x, 0)) if pulse else None
    _, ref = check_parity(name, T=T, B=B, C=C, p=p, mode="skip", x_fn=fn)
    if pulse:
        assert all(len(k) == 1 for k in ref.kept), [len(k) for k in ref.kept]


@pytest.mark.parametrize("name,how", [("tiny_conv", "zeros"), ("tiny_conv", "frozen"), ("vgg5", "zeros"),
                                      ("tiny_fc", "frozen")])
def test_tied_spike_sums(name, how):
    """Ties in s_t (reading 13: strict '>', ties skipped).  'zeros': an all-zero input keeps every layer silent,
    s_t = 0 for all t, every step ties the SST and only checkpoint rows are kept (all-zero gradients).
    'frozen': one input frame repeated, so s_t saturates into repeated values within a segment."""
    fn = (lambda x: np.zeros_like(x)) if how == "zeros" else (lambda x: np.repeat(x[:1], x.shape[0], axis=0))
    _, ref = check_parity(name, T=12 if name != "vgg5" else 14, B=2, C=2, p=40.0, mode="skip", x_fn=fn)
    if how == "zeros":
        assert (ref.s == 0).all() and all(len(k) == 1 for k in ref.kept)


@pytest.mark.parametrize("name,T,B,C,mode,group", [("tiny_conv", 24, 3, 4, "skip", 2), ("tiny_conv", 24, 3, 4, "ckpt", 3),
                                                  ("vgg5", 28, 2, 4, "skip", 4), ("tiny_resnet", 32, 2, 4, "skip", 2),
                                                  ("fc784", 20, 4, 2, "skip", 2), ("tiny_fc", 24, 3, 3, "skip", 3)])
def test_backward_groups(name, T, B, C, mode, group):
    """skipper_config.group = G: G segments recomputed into one arena and back-propagated as one layer-major pass
    (the reverse scan carries delta across the segment border as the per-segment carry does): the oracle's
    per-segment Skipper / checkpointed gradients, spikes of every recomputed row exact."""
    check_parity(name, T=T, B=B, C=C, p=50.0 if mode == "skip" else 0.0, mode=mode, group=group)


@pytest.mark.parametrize("name,T,B,C,mode", [("fc784", 64, 4, 1, "full"), ("tiny_fc", 40, 3, 1, "full"),
                                            ("tiny_fc", 48, 3, 2, "ckpt"), ("fc784", 60, 4, 3, "tbptt"),
                                            ("tiny_conv", 36, 2, 1, "full")])
def test_warp_parallel_fc_scan(name, T, B, C, mode):
    """The warp-parallel affine reverse scan of fc layers (lif_bwd_warp_kernel: 4 row chunks per neuron folded
    to (lam^len, partial) maps, composed with __shfl_sync, re-walked) on segments of >= 16 rows, against the
    oracle's serial Eq.2 recurrence."""
    check_parity(name, T=T, B=B, C=C, p=0.0, mode=mode)


@pytest.mark.parametrize("mode", ["full", "skip"])
def test_vgg5_reduced(mode):
    """cfg 2 topology (VGG-5) at reduced T and B: every kernel kind, several tiles, ragged tails."""
    check_parity("vgg5", T=14, B=2, C=2, p=40.0, mode=mode)


@pytest.mark.parametrize("name,T,B,mode,surrogate,gamma,pair,halo", [
    ("vgg5", 14, 3, "skip", "triangle", 0.3, "1", "1"), ("vgg5", 14, 3, "full", "fast_sigmoid", 1.0, "0", "1"),
    ("vgg5", 14, 3, "skip", "triangle", 0.3, "0", "0"), ("vgg5", 14, 2, "ckpt", "triangle", 0.3, "1", "0"),
    ("tiny_conv", 12, 3, "skip", "fast_sigmoid", 2.0, "1", "1"), ("vgg11", 24, 8, "skip", "triangle", 0.3, "1", "1")])
def test_fused_dgrad_reverse_scan(name, T, B, mode, surrogate, gamma, pair, halo, monkeypatch):
    """NEXT-1 backward half (conv_lif.cu BWD): the dgrad of a stride-1 conv layer with the previous layer's
    reverse surrogate scan (Eq.2) in its epilogue, forced on at reduced sizes (SKIPPER_CL_MIN_UNITS=0) for
    the CTA-pair / single-CTA and halo / per-tap producer variants and both surrogates (opt-in,
    SKIPPER_BWD_FUSION=1); the step matches the oracle and the fused class really ran."""
    monkeypatch.setenv("SKIPPER_BWD_FUSION", "1")
    monkeypatch.setenv("SKIPPER_CL_MIN_UNITS", "0")
    monkeypatch.setenv("SKIPPER_CL_PAIR", pair)
    monkeypatch.setenv("SKIPPER_CL_HALO", halo)
    check_parity(name, T=T, B=B, C=2, p=40.0, mode=mode, surrogate=surrogate, gamma=gamma)
    from paper_conf_micro_singhslsknnd22_b200 import SkipperNet
    net = synth.net_config(name)
    x, y = synth.make_inputs(net, T, B, seed=1)
    m = SkipperNet(net, T, C=2, p=40.0, mode=mode, batch=B, surrogate=surrogate, gamma=gamma)
    m.set_weights(synth.make_weights(net, seed=0))
    m.profile(True)
    m.step(torch.from_numpy(np.ascontiguousarray(x)).cuda(), torch.from_numpy(np.ascontiguousarray(y)).cuda())
    assert m.profile_read()["gemm_lif_bwd"]["launches"] > 0


def test_fused_dgrad_reverse_scan_single_row_segments(monkeypatch):
    """The fused dgrad + reverse scan on segments shrunk to K_c = 1 (one kept row per segment: the kernel's
    row walk is the carry in, one row, the carry out)."""
    monkeypatch.setenv("SKIPPER_BWD_FUSION", "1")
    monkeypatch.setenv("SKIPPER_CL_MIN_UNITS", "0")
    T, C = 24, 2
    S = T // C
    fn = lambda x: np.where((np.arange(x.shape[0]) % S == 0).reshape((-1,) + (1,) * (x.ndim - 1)), x, 0)  # noqa: E731
    check_parity("vgg5", T=T, B=2, C=C, p=95.0, mode="skip", x_fn=fn)


@pytest.mark.parametrize("pair", ["0", "1"])
def test_fused_dgrad_reverse_scan_bn64(pair, monkeypatch):
    """The 64-channel-tile variant of the fused dgrad + reverse scan (SKIPPER_CLB_BN64=1)."""
    monkeypatch.setenv("SKIPPER_BWD_FUSION", "1")
    monkeypatch.setenv("SKIPPER_CL_MIN_UNITS", "0")
    monkeypatch.setenv("SKIPPER_CLB_BN64", "1")
    monkeypatch.setenv("SKIPPER_CL_PAIR", pair)
    check_parity("vgg5", T=14, B=3, C=2, p=40.0, mode="skip")


@pytest.mark.parametrize("name,T,B,C,mode", [("vgg5", 14, 3, 2, "skip"), ("tiny_conv", 24, 3, 4, "ckpt"),
                                              ("tiny_resnet", 24, 2, 3, "skip"), ("tiny_fc", 24, 3, 6, "skip")])
def test_wgrad_overlap_slots(name, T, B, C, mode, monkeypatch):
    """SKIPPER_WGRAD_OVERLAP=1: the weight gradients' X operands alternate between two arena slots by
    segment parity and are no longer joined at each segment border - same gradients as the oracle."""
    monkeypatch.setenv("SKIPPER_WGRAD_OVERLAP", "1")
    check_parity(name, T=T, B=B, C=C, p=40.0, mode=mode)


@pytest.mark.parametrize("env", ["SKIPPER_L0_BWD_FUSION", "SKIPPER_NO_L0_FUSION", "SKIPPER_L0_CW32"])
def test_vgg5_layer0_variants(env, monkeypatch):
    """The alternative first-layer paths (fused reverse scan + wgrad; unfused im2col GEMM) agree too."""
    monkeypatch.setenv(env, "1")
    check_parity("vgg5", T=14, B=3, C=2, p=40.0, mode="skip")


def test_skip_p0_equals_ckpt_on_gpu():
    net = synth.net_config("tiny_conv")
    W = synth.make_weights(net)
    x, y = synth.make_inputs(net, 12, 2)
    m1, l1 = run_gpu(net, W, x, y, 12, 2, 0.0, "skip")
    m2, l2 = run_gpu(net, W, x, y, 12, 2, 0.0, "ckpt")
    assert l1 == l2 and m1.keep_mask().all()
    # same schedule, deterministic split-K weight gradients (slices summed in a fixed order): bitwise equal
    for a, b in zip(m1.grads(), m2.grads()):
        assert torch.equal(a, b)


@pytest.mark.parametrize("name,T,B,C,mode", [("vgg5", 20, 64, 2, "skip"), ("tiny_resnet", 16, 8, 2, "skip"),
                                            ("vgg5", 14, 16, 2, "full"), ("fc784", 20, 4, 2, "skip")])
def test_step_is_deterministic(name, T, B, C, mode):
    """Run-to-run determinism: the split-K weight gradients (tcgen05 GEMM slices, the
    narrow warp-MMA kernel's per-CTA slices) are summed in a fixed order, so two fresh contexts produce
    bitwise-identical gradients and post-Adam weights."""
    net = synth.net_config(name)
    W = synth.make_weights(net)
    x, y = synth.make_inputs(net, T, B)
    outs = []
    for _ in range(2):
        m, loss = run_gpu(net, W, x, y, T, C, 50.0 if mode == "skip" else 0.0, mode)
        outs.append((loss, [g.cpu() for g in m.grads()], [w.cpu() for w in m.weights()]))
        m.close()
    assert outs[0][0] == outs[1][0]
    for a, b in zip(outs[0][1] + outs[0][2], outs[1][1] + outs[1][2]):
        assert torch.equal(a, b)


def test_ckpt_equals_full_on_gpu():
    """Checkpointing reaches the BPTT gradient; same GEMM K-order -> bitwise or ~1e-6."""
    net = synth.net_config("tiny_conv")
    W = synth.make_weights(net)
    x, y = synth.make_inputs(net, 12, 2)
    m1, l1 = run_gpu(net, W, x, y, 12, 2, 0.0, "full")
    m2, l2 = run_gpu(net, W, x, y, 12, 2, 0.0, "ckpt")
    assert l1 == l2
    for a, b in zip(m1.grads(), m2.grads()):
        a, b = a.double(), b.double()
        assert (a - b).norm() <= 1e-5 * b.norm() + 1e-12


def test_segment_api_order_errors():
    from paper_conf_micro_singhslsknnd22_b200 import PASS_FIRST, PASS_RECOMPUTE, SkipperError, SkipperNet
    net = synth.net_config("tiny_fc")
    W = synth.make_weights(net)
    x, y = synth.make_inputs(net, 12, 2)
    m = SkipperNet(net, 12, C=2, p=50.0, mode="skip", batch=2)
    m.set_weights(W)
    xd, yd = torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda()
    with pytest.raises(SkipperError, match="EORDER"):
        m.forward_segment(1, PASS_FIRST, xd)
    with pytest.raises(SkipperError, match="EORDER"):
        m.backward_segment(1)
    m.forward_segment(0, PASS_FIRST, xd)
    m.forward_segment(1, PASS_FIRST, xd, yd)
    with pytest.raises(SkipperError, match="EORDER"):
        m.forward_segment(0, PASS_RECOMPUTE, xd)
    m.forward_segment(1, PASS_RECOMPUTE, xd)
    m.backward_segment(1)
    m.forward_segment(0, PASS_RECOMPUTE, xd)
    m.backward_segment(0)
    m.optimizer_step()


def test_memory_ordering_full_ckpt_skip():
    """Peak library memory: FULL > CKPT > SKIP on the same workload (Eq.3, Eq.6)."""
    net = synth.net_config("vgg5")
    W = synth.make_weights(net)
    T, B = 60, 4
    x, y = synth.make_inputs(net, T, B)
    peaks = {}
    for mode, C, p in [("full", 1, 0.0), ("ckpt", 6, 0.0), ("skip", 6, 40.0)]:
        m, _ = run_gpu(net, W, x, y, T, C, p, mode)
        peaks[mode] = m.mem_stats()[1]
        m.close()
    assert peaks["full"] > peaks["ckpt"] > peaks["skip"], peaks


@pytest.mark.parametrize("name,B", [("vgg5", 8), ("fc784", 64)])
def test_measured_peak_sublinear_in_T(name, B):
    """Eq.3 / Eq.6 on the device's allocator (not the analytic model): at C = sqrt(T) the peak device memory
    of CKPT and SKIP grows like sqrt(T) (x4 over a x16 range of T, plus T-independent weights / buffers)
    while FULL BPTT's grows linearly.  Covers the fc tail's chunked first pass."""
    from paper_conf_micro_singhslsknnd22_b200 import SkipperNet
    net = synth.net_config(name)
    W = synth.make_weights(net)
    Ts = (64, 256, 1024)
    x, y = synth.make_inputs(net, Ts[-1], B)
    xd, yd = torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda()
    peak = {}
    for mode, p in (("ckpt", 0.0), ("skip", 50.0), ("full", 0.0)):
        for T in Ts:
            C = int(round(T ** 0.5))
            m = SkipperNet(net, T, C=C, p=p, mode=mode, batch=B)
            m.set_weights(W)
            m.step(xd[:T].contiguous(), yd)
            peak[mode, T] = m.mem_stats()[1]
            m.close()
    # T grows x4 per point: stored state ~ sqrt(T) grows its INCREMENT x2 per point, linear growth x4 (the
    # T-independent part - weights, Adam moments, shadows, running state - cancels in the increments)
    inc = {mode: (peak[mode, Ts[2]] - peak[mode, Ts[1]]) / (peak[mode, Ts[1]] - peak[mode, Ts[0]])
           for mode in ("ckpt", "skip", "full")}
    print(name, {k: round(v / 1e6, 1) for k, v in peak.items()}, inc)
    assert inc["ckpt"] < 2.6 and inc["skip"] < 2.6, (inc, peak)
    assert inc["full"] > 3.0, (inc, peak)
    assert peak["skip", Ts[-1]] <= peak["ckpt", Ts[-1]] < peak["full", Ts[-1]], peak


@pytest.mark.parametrize("mode", ["skip", "full"])
def test_vgg11_reduced(mode):
    """cfg 3 topology (VGG-11: 8 conv incl. 256/512-channel layers down to 2x2, fc 512-4096-4096)."""
    check_parity("vgg11", T=24, B=2, C=2, p=50.0, mode=mode)


@pytest.mark.parametrize("name,T,B,C,p", [("tiny_conv", 20, 3, 2, 50.0), ("vgg5", 20, 2, 2, 40.0),
                                          ("fc784", 20, 4, 2, 50.0)])
def test_sam_weighted(name, T, B, C, p):
    """NEXT-2: the neuron-count-weighted SAM (reading 22) selects the same steps as the oracle."""
    check_parity(name, T=T, B=B, C=C, p=p, mode="skip", sam="weighted")


@pytest.mark.parametrize("mode,lam", [("full", 0.99), ("ckpt", 1.0), ("skip", 0.99), ("skip", 0.75)])
def test_tiny_resnet(mode, lam):
    """ResNet SNN pieces (reading 8, 23): stride-2 stem from DVS events, narrow im2col convs, identity and
    stride-2 / channel-padded option-A shortcuts, GAP readout."""
    check_parity("tiny_resnet", T=16, B=3, C=2, p=50.0, mode=mode, lam=lam)


@pytest.mark.parametrize("mode", ["skip", "full"])
def test_resnet20_dvs_reduced(mode):
    """cfg 4 topology (ResNet-20 SNN on 2x128x128 DVS frames) at reduced T and B: 19 spiking layers of
    every conv kind (im2col 16/32 channels, stride 2, implicit 64-channel, fused conv+LIF), 9 shortcuts."""
    check_parity("resnet20_dvs", T=44, B=1, C=2, p=50.0, mode=mode, deep=True)


def test_resnet20_dvs_gather_lif_32(monkeypatch):
    """SKIPPER_NO_NL32=1: the 32 -> 32 ResNet layers' fused conv + LIF on the tcgen05 gather kernel
    (conv_narrow.cu) instead of the default warp-level MMA kernel (narrow_lif.cu, two 16-channel K steps)."""
    monkeypatch.setenv("SKIPPER_NO_NL32", "1")
    check_parity("resnet20_dvs", T=44, B=1, C=2, p=50.0, mode="skip", deep=True)


@pytest.mark.parametrize("name,T,C", [("vgg5", 14, 2), ("tiny_resnet", 16, 2)])
def test_one_rank_nccl_bucketed_allreduce(name, T, C, monkeypatch):
    """K5 on the device: with a (one-rank) NCCL communicator the s allreduce and the bucketed dW
    allreduce on the comm stream run inside the step; the collectives are identities, so the
    gradients and post-Adam weights equal the communicator-free run."""
    from paper_conf_micro_singhslsknnd22_b200 import SkipperNet
    monkeypatch.setenv("SKIPPER_BUCKET_MB", "1")        # several buckets even for small nets
    net = synth.net_config(name)
    W = synth.make_weights(net)
    x, y = synth.make_inputs(net, T, 2)
    xd, yd = torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda()
    out = []
    for comm in (False, True):
        m = SkipperNet(net, T, C=C, p=50.0, mode="skip", batch=2)
        m.set_weights(W)
        if comm:
            m.comm_init(SkipperNet.comm_unique_id(), 0, 1)
        loss = m.step(xd, yd)
        out.append((loss, [g.cpu() for g in m.grads()], [w.cpu() for w in m.weights()], m.keep_mask()))
        m.close()
    assert out[0][0] == out[1][0]
    np.testing.assert_array_equal(out[0][3], out[1][3])
    # deterministic weight gradients and identity collectives: bitwise equal gradients and post-Adam weights
    for a, b in zip(out[0][1] + out[0][2], out[1][1] + out[1][2]):
        assert torch.equal(a, b)


@pytest.mark.parametrize("name,T,B,C,lam", [("tiny_fc", 12, 3, 3, 0.5), ("tiny_conv", 12, 3, 2, 0.99),
                                            ("vgg5", 14, 2, 2, None), ("tiny_resnet", 16, 3, 2, 0.75),
                                            ("fc784", 20, 4, 4, None)])
def test_tbptt(name, T, B, C, lam):
    """NEXT-4: truncated BPTT (Sec. III-C) on the device - per-window loss and readout, graph cut at window
    edges, state carried on - against the oracle (spikes exact, summed loss, dW)."""
    check_parity(name, T=T, B=B, C=C, p=0.0, mode="tbptt", lam=lam)


@pytest.mark.parametrize("name,T,B,C,p", [("tiny_conv", 20, 3, 2, 50.0), ("vgg5", 20, 2, 2, 40.0),
                                          ("fc784", 20, 4, 2, 50.0), ("tiny_resnet", 16, 2, 2, 50.0)])
def test_sam_l2trace(name, T, B, C, p):
    """NEXT-2, second variant: the l2 norm of the membrane trace per step (reading 25), accumulated inside every
    forward kernel (fused conv + LIF, layer 0, scans), selects the same steps as the oracle."""
    check_parity(name, T=T, B=B, C=C, p=p, mode="skip", sam="l2trace")


@pytest.mark.parametrize("T,B,shape,seed", [(7, 3, (32, 32, 3), 5), (20, 4, (784,), 123456789012),
                                            (5, 2, (128, 128, 2), 1)])
def test_poisson_encoder_bitexact(T, B, shape, seed):
    """NEXT-3: the device Poisson encoder draws the oracle's Philox4x32-10 numbers: spikes bit-exact."""
    from oracle.encoder import poisson_encode
    from paper_conf_micro_singhslsknnd22_b200 import encode_poisson
    rng = np.random.default_rng(seed % 1000)
    x = rng.random((B,) + shape, dtype=np.float32)
    rates = (0.5 + 0.5 * rng.random(T)).astype(np.float32)
    ref = poisson_encode(x.reshape(B, -1), rates, seed).reshape((T, B) + shape)
    out = encode_poisson(torch.from_numpy(x).cuda(), torch.from_numpy(rates).cuda(), seed).cpu().numpy()
    np.testing.assert_array_equal(out, ref)


def test_step_encoded_equals_step_on_encoded_spikes():
    """skipper_step_encoded / step_host_encoded = skipper_step on the oracle-encoded spikes (same loss, dW)."""
    from oracle.encoder import poisson_encode
    from paper_conf_micro_singhslsknnd22_b200 import SkipperNet
    net = synth.net_config("vgg5")
    W = synth.make_weights(net)
    T, B, seed = 14, 2, 99
    rng = np.random.default_rng(0)
    img = rng.random((B, 32, 32, 3), dtype=np.float32)
    rates = synth.envelope(np.arange(T)).astype(np.float32)
    x = poisson_encode(img.reshape(B, -1), rates, seed).reshape(T, B, 32, 32, 3)
    y = synth.labels(B, 10)
    ref = train_step(net, W, x, y, StepConfig(T=T, C=2, p=40.0, mode="skip"))
    out = []
    for how in ("spikes", "device", "host"):
        m = SkipperNet(net, T, C=2, p=40.0, mode="skip", batch=B)
        m.set_weights(W)
        if how == "spikes":
            loss = m.step(torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda())
        elif how == "device":
            loss = m.step_encoded(torch.from_numpy(img).cuda(), torch.from_numpy(rates).cuda(), seed,
                                  torch.from_numpy(y).cuda())
        else:
            loss = m.step_host_encoded(img, rates, seed, y)
        np.testing.assert_array_equal(m.spike_sums(), ref.s)
        out.append((loss, [g.cpu().numpy() for g in m.grads()]))
        m.close()
    for loss, grads in out:
        assert loss == pytest.approx(ref.loss, rel=1e-5)
        for g, r in zip(grads, ref.dW):
            ok, msg = grad_ok(g, r)
            assert ok, msg


# ---- BASELINE.json full sizes, in the configuration bench.py times (sampled outputs + properties)

def _full_size_gpu(wl):
    from paper_conf_micro_singhslsknnd22_b200 import SkipperNet
    net = synth.net_config(wl["net"])
    W = synth.make_weights(net)
    x, y = synth.make_inputs(net, wl["T"], wl["B"])
    m = SkipperNet(net, wl["T"], C=wl["C"], p=wl["p"], mode="skip", batch=wl["B"], debug_record=True)
    m.set_weights(W)
    loss = m.step(torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda())
    return net, W, x, y, m, loss


def _check_sampled(net, W, x, y, m, wl, samples, keep):
    """First-pass and recomputed states of sampled batch elements against the oracle run on those samples
    alone with the keep mask imposed (the recompute of a sample depends only on its input and the mask)."""
    spk = [L for L in net["layers"] if L["kind"] != "readout"]
    ref = train_step(net, W, np.ascontiguousarray(x[:, samples]), y[samples],
                     StepConfig(T=wl["T"], C=wl["C"], p=wl["p"], mode="skip", keep=keep, global_batch=wl["B"],
                                record=True))
    for l in range(len(spk)):
        for which, arr, exact in ((1, ref.first_o, True), (3, ref.rec_o, True), (0, ref.first_U, False),
                                  (2, ref.rec_U, False)):
            got = m.debug(which, l)[:, samples].cpu().numpy()
            if exact:
                assert np.array_equal(got, arr[l]), f"layer {l} debug {which}: {np.count_nonzero(got != arr[l])} differ"
            else:
                np.testing.assert_allclose(got, arr[l], rtol=1e-5, atol=1e-6)
    return ref


@pytest.mark.parametrize("name,samples", [("cfg2_vgg5", [0, 31, 63]), ("cfg4_resnet_dvs", [0, 31])])
def test_full_size_sampled_parity(name, samples):
    """cfg 2 (VGG-5, T=100, B=64, C=10, p=40) and cfg 4 (ResNet-20 DVS, T=300, B=32, C=5, p=50) at full size:
    s_t, per-layer counts, keep mask and loss against the oracle's full-batch first pass (computed in batch
    slices on the host cores); first-pass and recomputed spikes / membranes of sampled batch elements."""
    from _oracle_pool import full_batch_forward
    from oracle.bptt import readout
    from oracle.numerics import bf16_round
    from oracle.skipper import keep_mask
    wl = synth.workload(name)
    net, W, x, y, m, loss = _full_size_gpu(wl)
    counts, cnt = full_batch_forward(wl["net"], wl["T"], wl["B"], wl["C"])
    s = counts.sum(axis=0)
    np.testing.assert_array_equal(m.layer_spike_counts(), counts)
    np.testing.assert_array_equal(m.spike_sums(), s)
    keep = keep_mask(s, wl["T"], wl["C"], wl["p"])
    np.testing.assert_array_equal(m.keep_mask(), keep)
    ref_loss, _, _ = readout(bf16_round(W[-1]), cnt, y, wl["T"], wl["B"], bool(net["layers"][-1].get("gap")))
    assert loss == pytest.approx(ref_loss, rel=1e-5)
    _check_sampled(net, W, x, y, m, wl, samples, keep)
    m.close()


def test_full_size_vgg11_forward():
    """cfg 3 (VGG-11, T=200, B=128, C=5, p=50) at full size: s_t, per-layer counts, keep mask and loss against
    the oracle's full-batch first pass (batch slices on the host cores); first-pass and recomputed spikes /
    membranes of sampled batch elements against the oracle with its own mask imposed."""
    from _oracle_pool import full_batch_forward
    from oracle.bptt import readout
    from oracle.numerics import bf16_round
    from oracle.skipper import keep_mask
    wl = synth.workload("cfg3_vgg11")
    net, W, x, y, m, loss = _full_size_gpu(wl)
    counts, cnt = full_batch_forward(wl["net"], wl["T"], wl["B"], wl["C"])
    s = counts.sum(axis=0)
    np.testing.assert_array_equal(m.layer_spike_counts(), counts)
    np.testing.assert_array_equal(m.spike_sums(), s)
    keep = keep_mask(s, wl["T"], wl["C"], wl["p"])
    np.testing.assert_array_equal(m.keep_mask(), keep)
    assert 0 < keep.sum() < wl["T"]
    ref_loss, _, _ = readout(bf16_round(W[-1]), cnt, y, wl["T"], wl["B"], False)
    assert loss == pytest.approx(ref_loss, rel=1e-5)
    _check_sampled(net, W, x, y, m, wl, [0, 77, 127], keep)
    m.close()


@pytest.mark.parametrize("name,T,C,mode,env", [
    ("cfg2_vgg5", 0, 0, "skip", None), ("cfg2_vgg5", 0, 0, "full", None), ("cfg3_vgg11", 24, 2, "skip", None),
    ("cfg4_resnet_dvs", 0, 0, "skip", None),
    # the opt-in round-2 paths at full size: fused dgrad + reverse scan, two X-operand slots
    ("cfg2_vgg5", 0, 0, "skip", "SKIPPER_BWD_FUSION"), ("cfg3_vgg11", 24, 2, "skip", "SKIPPER_BWD_FUSION"),
    ("cfg2_vgg5", 0, 0, "skip", "SKIPPER_WGRAD_OVERLAP")])
def test_full_size_backward_parity(name, T, C, mode, env, monkeypatch):
    """Weight gradients at the BASELINE.json batch sizes in bench.py's launch configuration (no debug
    recording): cfg 2 at full size (T=100, B=64, C=10, p=40), cfg 3 at its full batch B=128 (the batch decides
    the kernel paths: fused conv+LIF, split-K counts of the fc GEMMs) with T=24, C=2, and cfg 4 at full size
    (T=300, B=32).  The oracle's dW is the sum of batch-slice training steps with the global keep mask (from its
    own full-batch first pass) and the global batch size imposed.  Tolerances as check_parity (cfg 4: deep)."""
    from _oracle_pool import full_batch_forward, full_batch_train
    from oracle.skipper import keep_mask
    from paper_conf_micro_singhslsknnd22_b200 import SkipperNet
    if env:
        monkeypatch.setenv(env, "1")
    wl = synth.workload(name)
    if T:
        wl["T"], wl["C"] = T, C
    net = synth.net_config(wl["net"])
    W = synth.make_weights(net)
    x, y = synth.make_inputs(net, wl["T"], wl["B"])
    m = SkipperNet(net, wl["T"], C=wl["C"], p=wl["p"], mode=mode, batch=wl["B"])
    m.set_weights(W)
    loss = m.step(torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda())
    grads = [g.cpu().numpy() for g in m.grads()]
    keep = None
    if mode == "skip":
        counts, _ = full_batch_forward(wl["net"], wl["T"], wl["B"], wl["C"])
        keep = keep_mask(counts.sum(axis=0), wl["T"], wl["C"], wl["p"])
        np.testing.assert_array_equal(m.keep_mask(), keep)
    m.close()
    dW, ref_loss = full_batch_train(wl["net"], wl["T"], wl["B"], wl["C"], wl["p"], mode, keep)
    assert loss == pytest.approx(ref_loss, rel=1e-5)
    deep = name.startswith("cfg4")
    tols = [(1e-3, 1e-3)] * len(dW)
    if deep:   # DESIGN.md §4 "deep networks": twice the bf16 contract's own effect, per layer
        exact, _ = full_batch_train(wl["net"], wl["T"], wl["B"], wl["C"], wl["p"], mode + "_exact", keep)
        tols = [(max(1e-3, 2 * grad_errs(b, a)[0]), max(1e-3, 2 * grad_errs(b, a)[1])) for a, b in zip(dW, exact)]
    report = []
    for l, (g, r) in enumerate(zip(grads, dW)):
        ok, msg = grad_ok(g, r, tols[l])
        report.append(f"layer {l}: {msg}")
        assert ok, f"layer {l} dW: {msg} (tolerance {tols[l][0]:.1e}, {tols[l][1]:.1e})"
    print(name, mode, "; ".join(report))
