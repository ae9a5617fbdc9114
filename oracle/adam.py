"""Adam ("Adam optimizer") - test infrastructure only.

The paper names Adam without hyper-parameters; reading 17: torch.optim.Adam
semantics, beta = (0.9, 0.999), eps = 1e-8, lr = 1e-3, no weight decay.
    m_t = b1 m + (1-b1) g ;  v_t = b2 v + (1-b2) g^2
    w  -= (lr / (1 - b1^t)) * m_t / (sqrt(v_t) / sqrt(1 - b2^t) + eps)
"""
from __future__ import annotations

import math

import numpy as np


def adam_update(w, g, m, v, step: int, lr=1e-3, beta1=0.9, beta2=0.999, eps=1e-8):
    """Returns (w, m, v) after one Adam step number `step` (1-based), float64."""
    w = np.asarray(w, np.float64)
    g = np.asarray(g, np.float64)
    m = beta1 * np.asarray(m, np.float64) + (1.0 - beta1) * g
    v = beta2 * np.asarray(v, np.float64) + (1.0 - beta2) * g * g
    bc1 = 1.0 - beta1 ** step
    bc2 = 1.0 - beta2 ** step
    denom = np.sqrt(v) / math.sqrt(bc2) + eps
    w = w - (lr / bc1) * m / denom
    return w, m, v
