"""bf16 rounding emulation (test infrastructure only; see oracle/__init__.py).

The GPU path feeds its tensor-core contractions with bf16 operands
(SURVEY.md §8(c) item 2 / reading 16).  The oracle emulates the rounding
round-to-nearest-even to 8 significant bits, directly from float64.
"""
from __future__ import annotations

import numpy as np


def bf16_round(a) -> np.ndarray:
    """Round to the nearest bf16 value (8 significant bits, ties to even).

    Definition: write a = m * 2**e with 0.5 <= |m| < 1 (frexp); the bf16 value is
    rint(m * 2**8) * 2**(e-8), np.rint being round-half-to-even.  Returned as
    float64 (every bf16 value is exact in float64).  Normal range only (the
    values on this path never approach bf16 over/underflow)."""
    a = np.asarray(a, dtype=np.float64)
    m, e = np.frexp(a)
    return np.ldexp(np.rint(m * 256.0), e - 8)
