"""Pins for the oracle's BPTT (Eq.2), checkpointing (Sec. V) and
Skipper (Sec. VI-A) against torch.autograd on an explicitly unrolled network.

The torch model below is written from Eq.1/Eq.2 independently of oracle/:
Heaviside spike with a surrogate backward, reset term detached ("the reset term
is not taken into account for the gradient computation"), torch's
own conv2d / avg_pool2d / cross_entropy.  Inputs are dyadic (lam in {1, .5, .75},
grid weights, small T) so the oracle's float32 forward equals the float64 one
exactly and the gradients must agree to ~1e-12."""
import numpy as np
import pytest
import torch
import torch.nn.functional as F

import synth
from oracle import StepConfig, train_step
from oracle.bptt import readout



class Spike(torch.autograd.Function):
    @staticmethod
    def forward(ctx, U, theta, gamma):
        ctx.save_for_backward(U)
        ctx.theta, ctx.gamma = theta, gamma
        return (U > theta).to(U.dtype)

    @staticmethod
    def backward(ctx, g):
        (U,) = ctx.saved_tensors
        sg = ctx.gamma * torch.clamp(1.0 - (U - ctx.theta).abs() / ctx.theta, min=0.0)
        return g * sg, None, None


def t_current(layer, W, a, a_res=None):
    """Synaptic current; ResNet layers (reading 8): stride, plus the option-A shortcut of the residual
    source written the classic CIFAR-ResNet way (subsample, zero-pad channels on both sides)."""
    if layer["kind"] == "conv":
        I = F.conv2d(a.permute(0, 3, 1, 2), W.permute(0, 3, 1, 2), padding=1,
                     stride=layer.get("stride", 1)).permute(0, 2, 3, 1)
        if a_res is not None:
            r = a_res.permute(0, 3, 1, 2)
            if r.shape[2] != I.shape[1]:
                r = r[:, :, ::2, ::2]
            pad = (I.shape[3] - r.shape[1]) // 2
            I = I + F.pad(r, (0, 0, 0, 0, pad, pad)).permute(0, 2, 3, 1)
        return I
    return a.reshape(a.shape[0], -1) @ W.T


def t_readin(net, cnt):
    if net["layers"][-1].get("gap"):
        return F.adaptive_avg_pool2d(cnt.permute(0, 3, 1, 2), 1).flatten(1)
    return cnt.reshape(cnt.shape[0], -1)


def t_out(layer, o):
    if layer["kind"] == "conv" and layer["pool"]:
        return F.avg_pool2d(o.permute(0, 3, 1, 2), 2).permute(0, 2, 3, 1)
    return o


def torch_full_bptt(net, W, x, y, gamma=0.3):
    spk = [L for L in net["layers"] if L["kind"] != "readout"]
    Wt = [torch.tensor(w.astype(np.float64), dtype=torch.float64, requires_grad=True) for w in W]
    T, B = x.shape[:2]
    U = [None] * len(spk)
    o = [None] * len(spk)
    cnt = 0
    for t in range(T):
        a = torch.tensor(x[t].astype(np.float64))
        outs = []
        for l, L in enumerate(spk):
            I = t_current(L, Wt[l], a, outs[L["res"]] if "res" in L else None)
            if U[l] is None:
                U[l] = I                                   # U_{-1} = o_{-1} = 0
            else:
                U[l] = L["lam"] * U[l] + I - L["theta"] * o[l].detach()
            o[l] = Spike.apply(U[l], L["theta"], gamma)
            a = t_out(L, o[l])
            outs.append(a)
        cnt = cnt + a
    z = t_readin(net, cnt) @ Wt[-1].T / T
    loss = F.cross_entropy(z, torch.tensor(y, dtype=torch.long), reduction="sum") / B
    loss.backward()
    return float(loss.detach()), [w.grad.numpy() for w in Wt]


def torch_skip_bptt(net, W, x, kept, dz, T, gamma=0.3):
    """Reading A of SURVEY.md §8(c) #14 as an autograd graph: within a segment the
    kept steps chain directly; the segment's first row carries the checkpoint
    value (from a no-grad first pass) with straight-through gradient paths to its
    own current I_{cS} and (times lam) to the previous segment's last kept U."""
    spk = [L for L in net["layers"] if L["kind"] != "readout"]
    Wt = [torch.tensor(w.astype(np.float64), dtype=torch.float64, requires_grad=True) for w in W]
    B = x.shape[1]
    # first pass, no grad: checkpoint states at each segment start
    ck = {}
    with torch.no_grad():
        U = [None] * len(spk)
        o = [None] * len(spk)
        starts = {int(k[0]) for k in kept}
        for t in range(T):
            a = torch.tensor(x[t].astype(np.float64))
            outs = []
            for l, L in enumerate(spk):
                I = t_current(L, Wt[l], a, outs[L["res"]] if "res" in L else None)
                U[l] = I if U[l] is None else L["lam"] * U[l] + I - L["theta"] * o[l]
                o[l] = (U[l] > L["theta"]).double()
                a = t_out(L, o[l])
                outs.append(a)
            if t in starts:
                ck[t] = [u.clone() for u in U]
    cnt = 0
    prev_last = None
    for rows in kept:
        U = [None] * len(spk)
        o = [None] * len(spk)
        for j, t in enumerate(rows):
            a = torch.tensor(x[t].astype(np.float64))
            outs = []
            for l, L in enumerate(spk):
                I = t_current(L, Wt[l], a, outs[L["res"]] if "res" in L else None)
                if j == 0:
                    u = ck[int(t)][l] + (I - I.detach())
                    if prev_last is not None:
                        u = u + L["lam"] * (prev_last[l] - prev_last[l].detach())
                    U[l] = u
                else:
                    U[l] = L["lam"] * U[l] + I - L["theta"] * o[l].detach()
                o[l] = Spike.apply(U[l], L["theta"], gamma)
                a = t_out(L, o[l])
                outs.append(a)
            cnt = cnt + a
        prev_last = list(U)
    z = t_readin(net, cnt) @ Wt[-1].T / T
    surrogate_loss = (torch.tensor(dz, dtype=torch.float64) * z).sum()
    surrogate_loss.backward()
    return [w.grad.numpy() for w in Wt]


def dyadic_setup(name, T, B, lam, seed=0):
    net = synth.net_config(name, lam=lam)
    W = synth.make_weights(net, seed=seed)
    x, y = synth.make_inputs(net, T, B, seed=seed + 1)
    return net, W, x, y


def rel_err(a, b):
    return np.linalg.norm(a - b) / max(np.linalg.norm(b), 1e-300)


@pytest.mark.parametrize("name,lam", [("tiny_fc", 1.0), ("tiny_fc", 0.5), ("tiny_conv", 0.75), ("tiny_conv", 1.0),
                                      ("tiny_resnet", 0.75), ("tiny_resnet", 1.0)])
def test_full_bptt_equals_autograd(name, lam):
    T = 6
    net, W, x, y = dyadic_setup(name, T, 3, lam)
    r = train_step(net, W, x, y, StepConfig(T=T, mode="full", emulate_bf16=False))
    loss, grads = torch_full_bptt(net, W, x, y)
    assert r.loss == pytest.approx(loss, rel=1e-12)
    assert any(np.abs(g).max() > 0 for g in grads[:-1]), "no gradient reached a spiking layer"
    for l, (a, b) in enumerate(zip(r.dW, grads)):
        assert rel_err(a, b) < 1e-12 or np.abs(a - b).max() < 1e-15, (l, rel_err(a, b))


@pytest.mark.parametrize("name,lam,C", [("tiny_fc", 0.5, 2), ("tiny_conv", 1.0, 3), ("tiny_resnet", 0.75, 2)])
def test_ckpt_equals_full_bitwise(name, lam, C):
    """Checkpointing reaches exactly the BPTT gradient."""
    T = 12
    net, W, x, y = dyadic_setup(name, T, 2, lam)
    rf = train_step(net, W, x, y, StepConfig(T=T, mode="full"))
    rc = train_step(net, W, x, y, StepConfig(T=T, C=C, mode="ckpt"))
    assert rf.loss == rc.loss
    for a, b in zip(rf.dW, rc.dW):
        np.testing.assert_array_equal(a, b)


def test_skip_p0_equals_ckpt_bitwise():
    T = 12
    net, W, x, y = dyadic_setup("tiny_conv", T, 2, 0.75)
    rc = train_step(net, W, x, y, StepConfig(T=T, C=3, mode="ckpt"))
    rs = train_step(net, W, x, y, StepConfig(T=T, C=3, mode="skip", p=0.0))
    assert rs.keep.all()
    for a, b in zip(rc.dW, rs.dW):
        np.testing.assert_array_equal(a, b)


@pytest.mark.parametrize("name,lam,C,seed", [("tiny_fc", 0.5, 1, 0), ("tiny_fc", 1.0, 3, 1),
                                             ("tiny_conv", 0.5, 2, 2), ("tiny_conv", 1.0, 1, 3),
                                             ("tiny_resnet", 0.5, 2, 4), ("tiny_resnet", 1.0, 3, 5)])
def test_skip_equals_autograd_on_compacted_chain(name, lam, C, seed):
    T = 12
    net, W, x, y = dyadic_setup(name, T, 2, lam, seed=seed)
    rng = np.random.default_rng(seed)
    keep = rng.random(T) < 0.6
    S = T // C
    keep[::S] = True
    r = train_step(net, W, x, y, StepConfig(T=T, C=C, mode="skip", p=50.0, keep=keep, emulate_bf16=False))
    grads = torch_skip_bptt(net, W, x, r.kept, r.dz, T)
    for l, (a, b) in enumerate(zip(r.dW, grads)):
        assert rel_err(a, b) < 1e-12 or np.abs(a - b).max() < 1e-15, (l, rel_err(a, b))


def test_skip_C1_reduces_to_full_on_compacted_input():
    """SURVEY.md §8(c) SKIP pin (ii): with C=1 and mask K, Skipper's gradient is
    full BPTT on x[K] with the first pass's dz and the original 1/T."""
    T = 14
    net, W, x, y = dyadic_setup("tiny_conv", T, 2, 0.75, seed=5)
    rng = np.random.default_rng(5)
    keep = rng.random(T) < 0.5
    keep[0] = True
    rs = train_step(net, W, x, y, StepConfig(T=T, C=1, mode="skip", p=30.0, keep=keep))
    K = np.nonzero(keep)[0]
    rf = train_step(net, W, x[K], y, StepConfig(T=len(K), mode="full", dz=rs.dz, T_norm=T))
    for a, b in zip(rs.dW, rf.dW):
        np.testing.assert_array_equal(a, b)


def test_skip_differs_from_ckpt_when_skipping():
    T = 20
    net, W, x, y = dyadic_setup("tiny_conv", T, 2, 0.99)
    rc = train_step(net, W, x, y, StepConfig(T=T, C=2, mode="ckpt"))
    rs = train_step(net, W, x, y, StepConfig(T=T, C=2, mode="skip", p=50.0))
    assert 0 < rs.keep.sum() < T
    assert not np.array_equal(rc.dW[0], rs.dW[0])
    assert rs.loss == rc.loss     # the loss comes from the full first pass


def test_readout_gradient_finite_differences():
    rng = np.random.default_rng(3)
    B, D, K, T = 3, 7, 5, 9
    WbL = rng.standard_normal((K, D))
    cnt = rng.integers(0, T + 1, (B, D)).astype(np.float64)
    y = rng.integers(0, K, B)
    loss, z, dz = readout(WbL, cnt, y, T, B)

    def f(zz):
        m = zz.max(1, keepdims=True)
        return float(((np.log(np.exp(zz - m).sum(1)) + m[:, 0]) - zz[np.arange(B), y]).sum() / B)
    assert f(z) == pytest.approx(loss, rel=1e-14)
    eps = 1e-6
    for b in range(B):
        for k in range(K):
            zp = z.copy()
            zp[b, k] += eps
            zm = z.copy()
            zm[b, k] -= eps
            assert (f(zp) - f(zm)) / (2 * eps) == pytest.approx(dz[b, k], abs=1e-8)


def test_bf16_emulation_changes_only_rounding():
    T = 8
    net, W, x, y = dyadic_setup("tiny_conv", T, 2, 1.0)
    r1 = train_step(net, W, x, y, StepConfig(T=T, mode="full"))
    r0 = train_step(net, W, x, y, StepConfig(T=T, mode="full", emulate_bf16=False))
    for a, b in zip(r1.dW[:-1], r0.dW[:-1]):
        assert rel_err(a, b) < 2e-2
    np.testing.assert_array_equal(r1.dW[-1], r0.dW[-1])


# ---- TBPTT (Sec. III-C; NEXT-4, reading 24)

def torch_tbptt(net, W, x, y, C, gamma=0.3):
    """Truncated BPTT as an autograd graph: the state carries on across windows but is detached at
    every window start; each window's loss is CE of its own readout integral / t'; loss = sum."""
    spk = [L for L in net["layers"] if L["kind"] != "readout"]
    Wt = [torch.tensor(w.astype(np.float64), dtype=torch.float64, requires_grad=True) for w in W]
    T, B = x.shape[:2]
    S = T // C
    U = [None] * len(spk)
    o = [None] * len(spk)
    total = 0
    for w in range(C):
        U = [u.detach() if u is not None else None for u in U]
        o = [v.detach() if v is not None else None for v in o]
        cnt = 0
        for t in range(w * S, (w + 1) * S):
            a = torch.tensor(x[t].astype(np.float64))
            outs = []
            for l, L in enumerate(spk):
                I = t_current(L, Wt[l], a, outs[L["res"]] if "res" in L else None)
                U[l] = I if U[l] is None else L["lam"] * U[l] + I - L["theta"] * o[l].detach()
                o[l] = Spike.apply(U[l], L["theta"], gamma)
                a = t_out(L, o[l])
                outs.append(a)
            cnt = cnt + a
        z = t_readin(net, cnt) @ Wt[-1].T / S
        total = total + F.cross_entropy(z, torch.tensor(y, dtype=torch.long), reduction="sum") / B
    total.backward()
    return float(total.detach()), [w.grad.numpy() for w in Wt]


@pytest.mark.parametrize("name,lam,C", [("tiny_fc", 0.5, 3), ("tiny_conv", 1.0, 2), ("tiny_resnet", 0.5, 2)])
def test_tbptt_equals_autograd(name, lam, C):
    T = 12
    net, W, x, y = dyadic_setup(name, T, 3, lam)
    r = train_step(net, W, x, y, StepConfig(T=T, C=C, mode="tbptt", emulate_bf16=False))
    loss, grads = torch_tbptt(net, W, x, y, C)
    assert r.loss == pytest.approx(loss, rel=1e-12)
    for l, (a, b) in enumerate(zip(r.dW, grads)):
        assert rel_err(a, b) < 1e-12 or np.abs(a - b).max() < 1e-15, (l, rel_err(a, b))


def test_tbptt_one_window_is_full_bptt():
    """t' = T (C = 1): TBPTT is plain BPTT."""
    T = 10
    net, W, x, y = dyadic_setup("tiny_conv", T, 2, 0.75)
    rt = train_step(net, W, x, y, StepConfig(T=T, C=1, mode="tbptt"))
    rf = train_step(net, W, x, y, StepConfig(T=T, mode="full"))
    assert rt.loss == rf.loss
    for a, b in zip(rt.dW, rf.dW):
        np.testing.assert_array_equal(a, b)


def test_tbptt_forward_state_is_not_truncated():
    """Only the gradient is truncated: the spikes of every window equal full BPTT's forward."""
    T = 12
    net, W, x, y = dyadic_setup("tiny_conv", T, 2, 0.75)
    rt = train_step(net, W, x, y, StepConfig(T=T, C=3, mode="tbptt", record=True))
    rf = train_step(net, W, x, y, StepConfig(T=T, mode="full", record=True))
    for a, b in zip(rt.first_o, rf.first_o):
        np.testing.assert_array_equal(a, b)
    np.testing.assert_array_equal(rt.s, rf.s)
    assert rt.ledger_peak * 3 == rf.ledger_peak      # one window of t' = T/3 stored at a time


# ---- the surrogate's threshold scaling and the fast-sigmoid branch (reading 4), pinned by autograd
# on the surrogate's ANTIDERIVATIVE: the spike is Heaviside in the forward value and F(U - theta) in the
# backward (straight-through, F - F.detach()), so torch differentiates F itself and nothing of sigma' is
# retyped here.  Triangle: F(x) = gamma (x - x|x| / (2 theta)) on |x| <= theta, constant outside, whose
# derivative is gamma max(0, 1 - |x| / theta).  Fast sigmoid: F(x) = x / (1 + kappa |x|), the fast sigmoid
# itself, whose derivative is 1 / (1 + kappa |x|)^2.

def st_spike(U, theta, kind, gamma):
    x = U - theta
    if kind == "triangle":
        xc = torch.clamp(x, -theta, theta)
        Fx = gamma * (xc - xc * xc.abs() / (2.0 * theta))
    else:
        Fx = x / (1.0 + gamma * x.abs())
    return (x > 0).to(U.dtype) + (Fx - Fx.detach())


def torch_full_bptt_st(net, W, x, y, kind, gamma):
    spk = [L for L in net["layers"] if L["kind"] != "readout"]
    Wt = [torch.tensor(w.astype(np.float64), dtype=torch.float64, requires_grad=True) for w in W]
    T, B = x.shape[:2]
    U = [None] * len(spk)
    o = [None] * len(spk)
    cnt = 0
    nspk = 0
    for t in range(T):
        a = torch.tensor(x[t].astype(np.float64))
        outs = []
        for l, L in enumerate(spk):
            I = t_current(L, Wt[l], a, outs[L["res"]] if "res" in L else None)
            U[l] = I if U[l] is None else L["lam"] * U[l] + I - L["theta"] * o[l].detach()
            o[l] = st_spike(U[l], L["theta"], kind, gamma)
            nspk += int(o[l].detach().sum())
            a = t_out(L, o[l])
            outs.append(a)
        cnt = cnt + a
    z = t_readin(net, cnt) @ Wt[-1].T / T
    loss = F.cross_entropy(z, torch.tensor(y, dtype=torch.long), reduction="sum") / B
    loss.backward()
    return float(loss.detach()), [w.grad.numpy() for w in Wt], nspk


@pytest.mark.parametrize("name,lam,theta,wscale,kind,gamma", [
    ("tiny_fc", 0.5, 2.0, 2.0, "triangle", 0.3),
    ("tiny_fc", 1.0, 0.5, 1.0, "triangle", 0.3),
    ("tiny_conv", 0.75, 2.0, 2.0, "triangle", 0.3),
    ("tiny_conv", 1.0, 0.5, 0.5, "triangle", 0.5),
    ("tiny_resnet", 0.75, 0.5, 1.0, "triangle", 0.3),
    ("tiny_fc", 0.5, 1.0, 1.0, "fast_sigmoid", 2.0),
    ("tiny_conv", 0.75, 2.0, 2.0, "fast_sigmoid", 4.0),
    ("tiny_resnet", 1.0, 0.5, 0.5, "fast_sigmoid", 1.0),
])
def test_full_bptt_surrogate_theta_and_kind_equal_autograd(name, lam, theta, wscale, kind, gamma):
    """theta != 1 and the fast-sigmoid surrogate: the oracle's sigma' (oracle/lif.py surrogate_grad) against
    autograd through the antiderivative.  Weights are scaled by a power of two (exact on the grid) so the
    network fires at theta != 1."""
    T = 6
    net = synth.net_config(name, lam=lam, theta=theta)
    W = [w * np.float32(wscale) if L["kind"] != "readout" else w for w, L in zip(synth.make_weights(net), net["layers"])]
    x, y = synth.make_inputs(net, T, 3, seed=1)
    r = train_step(net, W, x, y, StepConfig(T=T, mode="full", emulate_bf16=False, surrogate=kind, gamma=gamma))
    loss, grads, nspk = torch_full_bptt_st(net, W, x, y, kind, gamma)
    assert nspk > 0, "the network never fired"
    assert r.loss == pytest.approx(loss, rel=1e-12)
    assert all(np.abs(g).max() > 0 for g in grads[:-1]), "a spiking layer received no gradient"
    for l, (a, b) in enumerate(zip(r.dW, grads)):
        assert rel_err(a, b) < 1e-12 or np.abs(a - b).max() < 1e-15, (l, rel_err(a, b))


def test_st_spike_derivatives_match_reading4_shapes():
    """The antiderivatives above differentiate to reading 4's shapes at sample points (a check of the
    test's own F, so that the pin above is not vacuous)."""
    U = torch.linspace(-3.0, 5.0, 801, dtype=torch.float64, requires_grad=True)
    for theta in (0.5, 1.0, 2.0):
        g, = torch.autograd.grad(st_spike(U, theta, "triangle", 0.3).sum(), U)
        x = U.detach() - theta
        want = 0.3 * torch.clamp(1.0 - x.abs() / theta, min=0.0)
        assert torch.allclose(g, want, atol=1e-14)
        g, = torch.autograd.grad(st_spike(U, theta, "fast_sigmoid", 2.0).sum(), U)
        assert torch.allclose(g, 1.0 / (1.0 + 2.0 * x.abs()) ** 2, atol=1e-14)
