"""Poisson rate encoder with a counter-based generator - test infrastructure only (see oracle/__init__.py).

P:1165-1166 (reading 18): the input layer emits o0_t = [u_t < x * r_t], x the per-sample intensity in
[0, 1], r_t a rate envelope, u_t uniform in [0, 1).  NEXT-3 of SURVEY.md §8(f) moves this step onto the
device; both sides draw u from the same counter-based generator so the spikes can be compared bit for
bit: Philox4x32-10 (Salmon, Moraes, Dror, Shaw, SC'11), written out from its definition:
  round:  (hi0, lo0) = M0 * c0, (hi1, lo1) = M1 * c2 (32x32 -> 64 bit products)
          c <- (hi1 ^ c1 ^ k0, lo1, hi0 ^ c3 ^ k1, lo0);   k <- (k0 + W0, k1 + W1)   (mod 2^32)
  M0 = 0xD2511F53, M1 = 0xCD9E8D57, W0 = 0x9E3779B9, W1 = 0xBB67AE85; 10 rounds, the key bumped
  between rounds.  Element e of x_spikes[T][B][D] (row-major) uses word (e mod 4) of
  Philox(counter = (q mod 2^32, q div 2^32, 0, 0), key = (seed mod 2^32, seed div 2^32)), q = e div 4,
  and u = (word >> 8) * 2^-24 (exact in float32).  Comparison u < x * r_t in float32 (x * r_t rounded once).
"""
from __future__ import annotations

import numpy as np

M0, M1 = 0xD2511F53, 0xCD9E8D57
W0, W1 = 0x9E3779B9, 0xBB67AE85
MASK = 0xFFFFFFFF


def philox4x32_10(c0, c1, c2, c3, k0, k1):
    """Philox4x32-10 on uint64 arrays holding 32-bit values; returns the four output words."""
    c0, c1, c2, c3 = (np.asarray(v, np.uint64) & MASK for v in (c0, c1, c2, c3))
    k0 = np.uint64(k0 & MASK)
    k1 = np.uint64(k1 & MASK)
    for r in range(10):
        p0 = np.uint64(M0) * c0
        p1 = np.uint64(M1) * c2
        hi0, lo0 = p0 >> np.uint64(32), p0 & np.uint64(MASK)
        hi1, lo1 = p1 >> np.uint64(32), p1 & np.uint64(MASK)
        c0, c1, c2, c3 = hi1 ^ c1 ^ k0, lo1, hi0 ^ c3 ^ k1, lo0
        if r < 9:
            k0 = np.uint64((int(k0) + W0) & MASK)
            k1 = np.uint64((int(k1) + W1) & MASK)
    return c0, c1, c2, c3


def uniforms(n: int, seed: int) -> np.ndarray:
    """u_e for e = 0 .. n-1 (float32 in [0, 1), multiples of 2^-24)."""
    q = np.arange((n + 3) // 4, dtype=np.uint64)
    words = philox4x32_10(q & np.uint64(MASK), q >> np.uint64(32), 0, 0, seed & MASK, (seed >> 32) & MASK)
    w = np.stack(words, axis=1).reshape(-1)[:n]
    return ((w >> np.uint64(8)).astype(np.float64) * 2.0 ** -24).astype(np.float32)


def poisson_encode(x: np.ndarray, rates: np.ndarray, seed: int) -> np.ndarray:
    """x float32 [B][D] intensities, rates float32 [T] -> uint8 spikes [T][B][D] (o0_t = [u_t < x r_t])."""
    x = np.asarray(x, np.float32)
    rates = np.asarray(rates, np.float32)
    T = rates.shape[0]
    B, D = x.shape
    u = uniforms(T * B * D, seed).reshape(T, B, D)
    thr = (x[None, :, :] * rates[:, None, None]).astype(np.float32)
    return (u < thr).astype(np.uint8)
