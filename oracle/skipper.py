"""Skipper's time-skip policy and memory model - test infrastructure only.

SAM, Eq.4:    s_t = sum_{l=0}^{L_n} sum(o^l_t)
  reading 11: input spikes (l=0) plus every spiking layer's un-pooled spikes,
  over the global batch; the readout has no spikes.
SST, Eq.5:    SST_c = percentile({s_t : t in segment c}, p)
  reading 12: the segment's S = T/C values s_{cS..(c+1)S-1}; numpy 'linear'
  percentile in float64.
Keep rule: recompute t iff s_t > SST_c, otherwise skip.
  reading 9: t = cS is the checkpoint and is never skipped (Fig. 6 skips only
  within t in {1..9} and {11..19});
  reading 13: strict '>', and p == 0 keeps every step (SKIP(p=0) == CKPT).
Memory, Eq.3 ActCost = O(T/C) + O(C); Eq.6
  ActCost_skipper = O((1-p/100) T/C) + O(C); Eq.7 p/100 <= 1 - C*L_n/T.
"""
from __future__ import annotations

import numpy as np


def spike_sum_threshold(s: np.ndarray, T: int, C: int, p: float) -> np.ndarray:
    """SST_c for c = 0..C-1 (Eq.5), float64, via numpy.percentile(method='linear')."""
    S = T // C
    s = np.asarray(s, dtype=np.int64)
    return np.array([np.percentile(s[c * S:(c + 1) * S], p) for c in range(C)], dtype=np.float64)


def keep_mask(s: np.ndarray, T: int, C: int, p: float) -> np.ndarray:
    """bool[T]: True where timestep t is recomputed and back-propagated."""
    S = T // C
    keep = np.ones(T, dtype=bool)
    if p == 0:
        return keep
    sst = spike_sum_threshold(s, T, C, p)
    s = np.asarray(s, dtype=np.int64)
    for c in range(C):
        for t in range(c * S + 1, (c + 1) * S):
            keep[t] = s[t] > sst[c]
    return keep


def kept_lists(keep: np.ndarray, T: int, C: int) -> list:
    """Per segment, the ascending list of kept timesteps (always starting with cS)."""
    S = T // C
    return [np.nonzero(keep[c * S:(c + 1) * S])[0] + c * S for c in range(C)]


def ledger_model(mode: str, T: int, C: int, bytes_per_neuron_step: int, neurons: int,
                 kept_max: int | None = None) -> int:
    """Closed-form stored-state bytes at the peak (the Eq.3 / Eq.6 model).

    FULL stores every step; CKPT holds C checkpoints plus one
    segment of S = T/C steps (Eq.3); SKIP holds C checkpoints plus the largest
    kept set (Eq.6)."""
    per = bytes_per_neuron_step * neurons
    if mode == "full":
        return T * per
    S = T // C
    if mode == "ckpt":
        return (C + S) * per
    if mode == "skip":
        return (C + int(kept_max)) * per
    raise ValueError(mode)


def eq7_p_max(T: int, C: int, L_n: int) -> float:
    """Eq.7 rule of thumb: p/100 <= 1 - C*L_n/T."""
    return 100.0 * (1.0 - C * L_n / T)
