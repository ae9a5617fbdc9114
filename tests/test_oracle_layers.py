"""Pins for the oracle's contractions and pooling: brute-force loops, scipy
correlation, adjoint identities; bf16 rounding against torch."""
import numpy as np
import pytest
import scipy.signal
import torch

from oracle import bf16_round, conv3x3, conv3x3_input_grad, conv3x3_weight_grad, pool2, pool2_T


def brute_conv(a, W):
    N, H, Wd, Ci = a.shape
    Co = W.shape[0]
    out = np.zeros((N, H, Wd, Co))
    for n in range(N):
        for y in range(H):
            for x in range(Wd):
                for co in range(Co):
                    acc = 0.0
                    for dy in range(3):
                        for dx in range(3):
                            yy, xx = y + dy - 1, x + dx - 1
                            if 0 <= yy < H and 0 <= xx < Wd:
                                for ci in range(Ci):
                                    acc += W[co, dy, dx, ci] * a[n, yy, xx, ci]
                    out[n, y, x, co] = acc
    return out


@pytest.fixture
def rng():
    return np.random.default_rng(7)


def test_conv_brute_force(rng):
    a = rng.standard_normal((2, 5, 4, 3))
    W = rng.standard_normal((4, 3, 3, 3))
    np.testing.assert_allclose(conv3x3(a, W), brute_conv(a, W), rtol=1e-12, atol=1e-12)


def test_conv_scipy_correlate(rng):
    a = rng.standard_normal((2, 6, 7, 3))
    W = rng.standard_normal((5, 3, 3, 3))
    ref = np.zeros((2, 6, 7, 5))
    for n in range(2):
        for co in range(5):
            for ci in range(3):
                ref[n, :, :, co] += scipy.signal.correlate2d(a[n, :, :, ci], W[co, :, :, ci], mode="same")
    np.testing.assert_allclose(conv3x3(a, W), ref, rtol=1e-12, atol=1e-12)


def test_conv_adjoints(rng):
    a = rng.standard_normal((3, 6, 4, 5))
    W = rng.standard_normal((7, 3, 3, 5))
    d = rng.standard_normal((3, 6, 4, 7))
    lhs = np.sum(conv3x3(a, W) * d)
    assert np.sum(a * conv3x3_input_grad(d, W)) == pytest.approx(lhs, rel=1e-12)
    assert np.sum(W * conv3x3_weight_grad(d, a)) == pytest.approx(lhs, rel=1e-12)


def test_conv_torch(rng):
    a = rng.standard_normal((2, 8, 8, 4))
    W = rng.standard_normal((6, 3, 3, 4))
    ref = torch.nn.functional.conv2d(torch.tensor(a).permute(0, 3, 1, 2),
                                     torch.tensor(W).permute(0, 3, 1, 2), padding=1).permute(0, 2, 3, 1)
    np.testing.assert_allclose(conv3x3(a, W), ref.numpy(), rtol=1e-12, atol=1e-12)


def test_pool_brute_and_adjoint(rng):
    o = (rng.random((2, 6, 4, 3)) < 0.4).astype(np.uint8)
    p = pool2(o)
    for n in range(2):
        for y in range(3):
            for x in range(2):
                for c in range(3):
                    assert p[n, y, x, c] == (o[n, 2 * y, 2 * x, c] + o[n, 2 * y + 1, 2 * x, c]
                                             + o[n, 2 * y, 2 * x + 1, c] + o[n, 2 * y + 1, 2 * x + 1, c]) / 4
    assert set(np.unique(p)) <= {0, 0.25, 0.5, 0.75, 1.0}
    g = rng.standard_normal(p.shape)
    assert np.sum(p * g) == pytest.approx(np.sum(o * pool2_T(g)), rel=1e-12)


def test_bf16_round_matches_torch(rng):
    x = (rng.standard_normal(200000) * np.exp(rng.uniform(-20, 20, 200000))).astype(np.float32)
    # add exact ties: 8 significant bits + a half ulp
    ties = (np.arange(1, 2001, dtype=np.float64) * 2 + 1) * 2.0 ** -10
    x = np.concatenate([x, ties.astype(np.float32), -ties.astype(np.float32)])
    ref = torch.tensor(x).to(torch.bfloat16).to(torch.float64).numpy()
    np.testing.assert_array_equal(bf16_round(x.astype(np.float64)), ref)


def test_bf16_grid_values_exact(rng):
    j = rng.integers(-255, 256, 1000)
    w = j * 2.0 ** -9
    np.testing.assert_array_equal(bf16_round(w), w)


# ---- ResNet pieces (reading 8, reading 23): strided conv, option-A shortcut, global average pool

def brute_conv_strided(a, W, s):
    N, H, Wd, Ci = a.shape
    Co = W.shape[0]
    Ho, Wo = (H + s - 1) // s, (Wd + s - 1) // s
    out = np.zeros((N, Ho, Wo, Co))
    for n in range(N):
        for y in range(Ho):
            for x in range(Wo):
                for dy in range(3):
                    for dx in range(3):
                        yy, xx = s * y + dy - 1, s * x + dx - 1
                        if 0 <= yy < H and 0 <= xx < Wd:
                            out[n, y, x] += W[:, dy, dx, :] @ a[n, yy, xx, :]
    return out


@pytest.mark.parametrize("shape", [(2, 8, 8, 3), (1, 6, 10, 2), (2, 5, 7, 4)])
def test_conv_stride2_brute_and_torch(rng, shape):
    a = rng.standard_normal(shape)
    W = rng.standard_normal((5, 3, 3, shape[3]))
    out = conv3x3(a, W, 2)
    np.testing.assert_allclose(out, brute_conv_strided(a, W, 2), rtol=1e-12, atol=1e-12)
    ref = torch.nn.functional.conv2d(torch.tensor(a).permute(0, 3, 1, 2), torch.tensor(W).permute(0, 3, 1, 2),
                                     padding=1, stride=2).permute(0, 2, 3, 1)
    np.testing.assert_allclose(out, ref.numpy(), rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("stride", [1, 2])
def test_conv_strided_adjoints(rng, stride):
    a = rng.standard_normal((2, 8, 6, 3))
    W = rng.standard_normal((4, 3, 3, 3))
    y = conv3x3(a, W, stride)
    d = rng.standard_normal(y.shape)
    lhs = np.sum(y * d)
    assert np.sum(a * conv3x3_input_grad(d, W, stride, a.shape[1:3])) == pytest.approx(lhs, rel=1e-12)
    assert np.sum(W * conv3x3_weight_grad(d, a, stride)) == pytest.approx(lhs, rel=1e-12)


def test_shortcut_option_a(rng):
    from oracle.layers import shortcut_a, shortcut_a_T
    a = (rng.random((2, 8, 8, 4)) < 0.5).astype(np.float64)
    s = shortcut_a(a, 2, 8)                       # 4 -> 8 channels, 2 zero channels each side
    assert s.shape == (2, 4, 4, 8)
    np.testing.assert_array_equal(s[..., :2], 0)
    np.testing.assert_array_equal(s[..., 6:], 0)
    for y in range(4):
        for x in range(4):
            np.testing.assert_array_equal(s[:, y, x, 2:6], a[:, 2 * y, 2 * x, :])
    # the classic CIFAR ResNet option-A: F.pad(x[:, :, ::2, ::2], (0, 0, 0, 0, c/4, c/4)) in NCHW
    ref = torch.nn.functional.pad(torch.tensor(a).permute(0, 3, 1, 2)[:, :, ::2, ::2], (0, 0, 0, 0, 2, 2))
    np.testing.assert_array_equal(s, ref.permute(0, 2, 3, 1).numpy())
    np.testing.assert_array_equal(shortcut_a(a, 1, 4), a)                     # identity shortcut
    g = rng.standard_normal(s.shape)
    assert np.sum(s * g) == pytest.approx(np.sum(a * shortcut_a_T(g, 2, 4, (8, 8))), rel=1e-12)


def test_gap_and_adjoint(rng):
    from oracle.layers import gap, gap_T
    o = (rng.random((3, 4, 4, 5)) < 0.3).astype(np.uint8)
    p = gap(o)
    np.testing.assert_array_equal(p * 16, o.sum(axis=(1, 2)))
    g = rng.standard_normal(p.shape)
    assert np.sum(p * g) == pytest.approx(np.sum(o * gap_T(g, (4, 4))), rel=1e-12)
