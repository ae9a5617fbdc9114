"""LIF neuron (Eq.1) and surrogate derivative (Eq.2) - test infrastructure only.

Eq.1 (reconstructed in SURVEY.md §0.1):
    U^l_t = lam * U^l_{t-1} + W^l o^{l-1}_t - theta * o^l_{t-1}
    o^l_t = 1 if U^l_t > theta else 0
Readings: the reset term sits outside the leak (#1), the
threshold is strict (#2), U_{-1} = 0 and o_{-1} = 0 (#3).

Eq.2: sigma' is "the smooth surrogate function" and "the
reset term is not taken into account for the gradient computation".
Reading #4: triangle sigma'(U) = gamma * max(0, 1 - |U - theta| / theta),
gamma = 0.3; fast-sigmoid 1/(1 + kappa |U - theta|)^2 selectable.
"""
from __future__ import annotations

import numpy as np


def lif_step(U_prev: np.ndarray, o_prev: np.ndarray, I: np.ndarray, lam: float, theta: float):
    """One Eq.1 update in float32, no fused multiply-add, order ((lam*U) + I) - theta*o.

    U_prev, I: float32 arrays; o_prev: {0,1} array.  Returns (U float32, o uint8)."""
    lam32 = np.float32(lam)
    th32 = np.float32(theta)
    U_prev = np.asarray(U_prev, np.float32)
    I = np.asarray(I, np.float32)
    leak = lam32 * U_prev                       # float32 product, rounded
    integ = leak + I                            # float32 sum, rounded
    reset = th32 * np.asarray(o_prev, np.float32)  # exact: theta or 0
    U = integ - reset                           # float32 difference, rounded
    o = (U > th32).astype(np.uint8)
    return U, o


def surrogate_grad(U: np.ndarray, theta: float, kind: str = "triangle", gamma: float = 0.3) -> np.ndarray:
    """sigma'(U) in float64 (Eq.2, reading 4)."""
    U = np.asarray(U, np.float64)
    th = float(theta)
    if kind == "triangle":
        return gamma * np.maximum(0.0, 1.0 - np.abs(U - th) / th)
    if kind == "fast_sigmoid":
        return 1.0 / (1.0 + gamma * np.abs(U - th)) ** 2
    raise ValueError(f"unknown surrogate {kind!r}")
