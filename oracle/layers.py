"""Synaptic contractions and pooling (test infrastructure only; see oracle/__init__.py).

The paper's networks (Table I) use conv and linear layers; it
does not fix padding or pooling.  Readings: 3x3 convolution,
zero padding 1, no bias (Eq.1 has none), stride 1 or 2 (the
ResNet20 SNN of Table I downsamples; reading 8); 2x2 average pooling of output
spikes (reading 7); ResNet shortcuts are option A (spatial subsample +
channel zero pad, no parameters; reading 8); global average pooling feeds the
ResNet readout (reading 23).  Layout NHWC; weights [Cout][3][3][Cin].
All in float64.
"""
from __future__ import annotations

import numpy as np


def conv3x3(a: np.ndarray, W: np.ndarray, stride: int = 1) -> np.ndarray:
    """out[n,y,x,co] = sum_{dy,dx,ci} W[co,dy,dx,ci] * a[n, s*y+dy-1, s*x+dx-1, ci] (zero outside),
    output size ceil(H/s) x ceil(W/s).

    Written as one matmul per tap over the zero-padded input."""
    N, H, Wd, Ci = a.shape
    Co = W.shape[0]
    Ho, Wo = -(-H // stride), -(-Wd // stride)
    ap = np.pad(np.asarray(a, np.float64), ((0, 0), (1, 1 + stride), (1, 1 + stride), (0, 0)))
    out = np.zeros((N, Ho, Wo, Co), dtype=np.float64)
    for dy in range(3):
        for dx in range(3):
            win = ap[:, dy:dy + stride * Ho:stride, dx:dx + stride * Wo:stride, :]
            out += win @ np.asarray(W[:, dy, dx, :], np.float64).T
    return out


def conv3x3_input_grad(d: np.ndarray, W: np.ndarray, stride: int = 1, in_hw: tuple | None = None) -> np.ndarray:
    """Adjoint of conv3x3 in its input (in_hw = the input's H, W; default the output's times s):
    ga[n,yi,xi,ci] = sum over (y, x, dy, dx) with s*y+dy-1 = yi, s*x+dx-1 = xi of W[co,dy,dx,ci] d[n,y,x,co].

    Written as a scatter of one matmul per tap into the zero-padded input."""
    N, Ho, Wo, Co = d.shape
    Ci = W.shape[3]
    H, Wd = in_hw if in_hw is not None else (Ho * stride, Wo * stride)
    gp = np.zeros((N, H + 2 + stride, Wd + 2 + stride, Ci), dtype=np.float64)
    d64 = np.asarray(d, np.float64)
    for dy in range(3):
        for dx in range(3):
            gp[:, dy:dy + stride * Ho:stride, dx:dx + stride * Wo:stride, :] += d64 @ np.asarray(W[:, dy, dx, :], np.float64)
    return gp[:, 1:1 + H, 1:1 + Wd, :]


def conv3x3_weight_grad(d: np.ndarray, a: np.ndarray, stride: int = 1) -> np.ndarray:
    """Adjoint of conv3x3 in its weights:
    gW[co,dy,dx,ci] = sum_{n,y,x} d[n,y,x,co] * a[n, s*y+dy-1, s*x+dx-1, ci]."""
    N, Ho, Wo, Co = d.shape
    Ci = a.shape[3]
    ap = np.pad(np.asarray(a, np.float64), ((0, 0), (1, 1 + stride), (1, 1 + stride), (0, 0)))
    d2 = np.asarray(d, np.float64).reshape(-1, Co)
    out = np.zeros((Co, 3, 3, Ci), dtype=np.float64)
    for dy in range(3):
        for dx in range(3):
            win = ap[:, dy:dy + stride * Ho:stride, dx:dx + stride * Wo:stride, :]
            out[:, dy, dx, :] = d2.T @ win.reshape(-1, Ci)
    return out


def shortcut_a(a: np.ndarray, stride: int, cout: int) -> np.ndarray:
    """Option-A ResNet shortcut (reading 8): out[n,y,x,c] = a[n, s*y, s*x, c - lo] for
    lo <= c < lo + Cin with lo = (cout - Cin) // 2, zero elsewhere (no parameters)."""
    N, H, Wd, Ci = a.shape
    lo = (cout - Ci) // 2
    sub = np.asarray(a, np.float64)[:, ::stride, ::stride, :]
    out = np.zeros(sub.shape[:3] + (cout,), dtype=np.float64)
    out[..., lo:lo + Ci] = sub
    return out


def shortcut_a_T(g: np.ndarray, stride: int, cin: int, in_hw: tuple) -> np.ndarray:
    """Adjoint of shortcut_a: the channel window lo..lo+cin of g scattered back to the subsampled positions."""
    N, Ho, Wo, Co = g.shape
    lo = (Co - cin) // 2
    out = np.zeros((N,) + tuple(in_hw) + (cin,), dtype=np.float64)
    out[:, ::stride, ::stride, :] = np.asarray(g, np.float64)[..., lo:lo + cin]
    return out


def gap(a: np.ndarray) -> np.ndarray:
    """Global average pooling over (h, w) of an NHWC array (reading 23)."""
    return np.asarray(a, np.float64).mean(axis=(1, 2))


def gap_T(g: np.ndarray, hw: tuple) -> np.ndarray:
    """Adjoint of gap: g / (h w) broadcast over every position."""
    H, Wd = hw
    g = np.asarray(g, np.float64) / (H * Wd)
    return np.broadcast_to(g[:, None, None, :], (g.shape[0], H, Wd, g.shape[1])).copy()


def pool2(o: np.ndarray) -> np.ndarray:
    """2x2 average pooling, stride 2 (reading 7): values of spikes -> {0, .25, .5, .75, 1}."""
    N, H, Wd, C = o.shape
    return np.asarray(o, np.float64).reshape(N, H // 2, 2, Wd // 2, 2, C).mean(axis=(2, 4))


def pool2_T(g: np.ndarray) -> np.ndarray:
    """Adjoint of pool2: each pooled gradient is spread as g/4 over its 2x2 window."""
    N, h, w, C = g.shape
    g = np.asarray(g, np.float64) * 0.25
    return np.repeat(np.repeat(g, 2, axis=1), 2, axis=2)
