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
SAM variants (NEXT-2, "the sum of spike counts weighted by the neuron count in each
layer"): reading 22 - 'weighted' divides each layer's count by its neurons per sample (l = 0 is the
input), s_t = sum_l count_l,t / N_l in float64, summed in layer order l = 0..L_n (per-layer firing
rates, so small layers weigh as much as large ones).  The default 'spikes' is Eq.4.
Memory, Eq.3 ActCost = O(T/C) + O(C); Eq.6
  ActCost_skipper = O((1-p/100) T/C) + O(C); Eq.7 p/100 <= 1 - C*L_n/T.
"""
from __future__ import annotations

import numpy as np


def _metric(s):
    """SAM values as given: integer spike sums stay int64, fractional metrics float64."""
    s = np.asarray(s)
    return s.astype(np.int64) if np.issubdtype(s.dtype, np.integer) else s.astype(np.float64)


def sam_weighted(counts: np.ndarray, neurons) -> np.ndarray:
    """NEXT-2 metric (reading 22): counts int64 [L_n + 1][T] (row 0 = input spikes), neurons per
    sample of each row -> s_t = sum_l counts[l][t] / neurons[l], float64, accumulated in l order."""
    counts = np.asarray(counts, np.int64)
    s = np.zeros(counts.shape[1], np.float64)
    for l in range(counts.shape[0]):
        s = s + counts[l].astype(np.float64) / float(neurons[l])
    return s


def spike_sum_threshold(s: np.ndarray, T: int, C: int, p: float) -> np.ndarray:
    """SST_c for c = 0..C-1 (Eq.5), float64, via numpy.percentile(method='linear')."""
    S = T // C
    s = _metric(s)
    return np.array([np.percentile(s[c * S:(c + 1) * S], p) for c in range(C)], dtype=np.float64)


def keep_mask(s: np.ndarray, T: int, C: int, p: float) -> np.ndarray:
    """bool[T]: True where timestep t is recomputed and back-propagated."""
    S = T // C
    keep = np.ones(T, dtype=bool)
    if p == 0:
        return keep
    sst = spike_sum_threshold(s, T, C, p)
    s = _metric(s)
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
