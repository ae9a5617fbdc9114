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
