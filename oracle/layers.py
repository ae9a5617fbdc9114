"""Synaptic contractions and pooling (test infrastructure only; see oracle/__init__.py).

The paper's networks (Table I) use conv and linear layers; it
does not fix padding or pooling.  Readings: 3x3 convolution,
stride 1, zero padding 1, no bias (Eq.1 has none); 2x2 average
pooling of output spikes (reading 7).  Layout NHWC; weights [Cout][3][3][Cin].
All in float64.
"""
from __future__ import annotations

import numpy as np


def conv3x3(a: np.ndarray, W: np.ndarray) -> np.ndarray:
    """out[n,y,x,co] = sum_{dy,dx,ci} W[co,dy,dx,ci] * a[n, y+dy-1, x+dx-1, ci] (zero outside).

    Written as one matmul per tap over the zero-padded input."""
    N, H, Wd, Ci = a.shape
    Co = W.shape[0]
    ap = np.pad(np.asarray(a, np.float64), ((0, 0), (1, 1), (1, 1), (0, 0)))
    out = np.zeros((N, H, Wd, Co), dtype=np.float64)
    for dy in range(3):
        for dx in range(3):
            out += ap[:, dy:dy + H, dx:dx + Wd, :] @ np.asarray(W[:, dy, dx, :], np.float64).T
    return out


def conv3x3_input_grad(d: np.ndarray, W: np.ndarray) -> np.ndarray:
    """Adjoint of conv3x3 in its input:
    ga[n,y,x,ci] = sum_{dy,dx,co} W[co,dy,dx,ci] * d[n, y-dy+1, x-dx+1, co]."""
    N, H, Wd, Co = d.shape
    Ci = W.shape[3]
    dp = np.pad(np.asarray(d, np.float64), ((0, 0), (1, 1), (1, 1), (0, 0)))
    out = np.zeros((N, H, Wd, Ci), dtype=np.float64)
    for dy in range(3):
        for dx in range(3):
            out += dp[:, 2 - dy:2 - dy + H, 2 - dx:2 - dx + Wd, :] @ np.asarray(W[:, dy, dx, :], np.float64)
    return out


def conv3x3_weight_grad(d: np.ndarray, a: np.ndarray) -> np.ndarray:
    """Adjoint of conv3x3 in its weights:
    gW[co,dy,dx,ci] = sum_{n,y,x} d[n,y,x,co] * a[n, y+dy-1, x+dx-1, ci]."""
    N, H, Wd, Co = d.shape
    Ci = a.shape[3]
    ap = np.pad(np.asarray(a, np.float64), ((0, 0), (1, 1), (1, 1), (0, 0)))
    d2 = np.asarray(d, np.float64).reshape(-1, Co)
    out = np.zeros((Co, 3, 3, Ci), dtype=np.float64)
    for dy in range(3):
        for dx in range(3):
            out[:, dy, dx, :] = d2.T @ ap[:, dy:dy + H, dx:dx + Wd, :].reshape(-1, Ci)
    return out


def pool2(o: np.ndarray) -> np.ndarray:
    """2x2 average pooling, stride 2 (reading 7): values of spikes -> {0, .25, .5, .75, 1}."""
    N, H, Wd, C = o.shape
    return np.asarray(o, np.float64).reshape(N, H // 2, 2, Wd // 2, 2, C).mean(axis=(2, 4))


def pool2_T(g: np.ndarray) -> np.ndarray:
    """Adjoint of pool2: each pooled gradient is spread as g/4 over its 2x2 window."""
    N, h, w, C = g.shape
    g = np.asarray(g, np.float64) * 0.25
    return np.repeat(np.repeat(g, 2, axis=1), 2, axis=2)
