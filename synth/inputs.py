"""Seeded input generators (no method arithmetic; see synth/__init__.py).

Seeds: weights 0, inputs 1, labels 2 unless overridden.
"""
from __future__ import annotations

import math

import numpy as np

JMAX = 255  # |j| <= 255: every grid weight is exact in bf16 (8 significant bits)


def _layer_fan_in(layer) -> int:
    return layer["cin"] * (9 if layer["kind"] == "conv" else 1)


def weight_shape(layer) -> tuple:
    if layer["kind"] == "conv":
        return (layer["cout"], 3, 3, layer["cin"])
    return (layer["cout"], layer["cin"])


def grid_weights(layer, rng: np.random.Generator, rate_in: float, gain: float = 0.45,
                 bias: float = 0.15) -> np.ndarray:
    """Weights on the dyadic grid j * 2**-e (SURVEY.md §8(c) exactness protocol).

    j ~ round(Normal(bias*64, 64)) clipped to [-255, 255]; the exponent e is
    picked from the fan-in so that the synaptic current has a standard
    deviation of about `gain` (in units of theta) for inputs firing at
    `rate_in`.  Returned as float32 (every value exact).
    """
    fan_in = _layer_fan_in(layer)
    sigma_w = gain / math.sqrt(fan_in * max(rate_in, 1e-3))
    sigma_j = 64.0
    e = int(round(math.log2(sigma_j / sigma_w)))
    j = np.rint(rng.normal(bias * sigma_j, sigma_j, size=weight_shape(layer)))
    j = np.clip(j, -JMAX, JMAX)
    return (j * 2.0 ** (-e)).astype(np.float32)


def make_weights(net, seed: int = 0, gain: float = 0.6, bias: float = 0.0):
    """One float32 master weight array per layer (spiking layers and readout)."""
    rng = np.random.default_rng(seed)
    out = []
    # input firing rate: Poisson frames ~0.37 (envelope mean ~0.75 * E[x]=0.5); DVS events ~0.02
    rate = 0.02 if net.get("input", ("",))[0] == "dvs" else 0.3
    for layer in net["layers"]:
        if layer["kind"] == "readout":
            out.append(grid_weights(layer, rng, rate_in=rate, gain=2.0, bias=0.0))
        else:
            out.append(grid_weights(layer, rng, rate_in=rate, gain=gain, bias=bias))
            rate = 0.12
    return out


def envelope(t: np.ndarray | int, period: float = 25.0) -> np.ndarray:
    """Temporal rate envelope r_t = 0.5 + 0.5*sin^2(pi t / period) (SURVEY.md §8(d) cfg 2).

    Makes the spike activity s_t non-stationary so that the SAM percentile
    has something to select."""
    t = np.asarray(t, dtype=np.float64)
    return 0.5 + 0.5 * np.sin(np.pi * t / period) ** 2


def poisson_frames(T: int, B: int, shape: tuple, seed: int = 1, rate_scale: float = 1.0,
                   use_envelope: bool = True) -> np.ndarray:
    """Poisson rate coding o0_t = [u_t < x * r_t] (reading 18).

    x ~ U[0,1]^shape per sample (fixed over time), u_t ~ U[0,1) fresh each step.
    Returns uint8 {0,1} of shape [T][B][*shape]."""
    rng = np.random.default_rng(seed)
    x = rng.random((B,) + tuple(shape), dtype=np.float32) * np.float32(rate_scale)
    out = np.empty((T, B) + tuple(shape), dtype=np.uint8)
    for t in range(T):
        r = np.float32(envelope(t)) if use_envelope else np.float32(1.0)
        u = rng.random((B,) + tuple(shape), dtype=np.float32)
        out[t] = (u < x * r)
    return out


def dvs_frames(T: int, B: int, H: int = 128, W: int = 128, seed: int = 1) -> np.ndarray:
    """DVS-Gesture-shaped event frames u8 [T][B][H][W][2] (SURVEY.md §8(d) cfg 4).

    Bernoulli events at ~1-3 % per pixel-polarity per step, concentrated in a
    Gaussian blob that moves along a circle, with a burst envelope."""
    rng = np.random.default_rng(seed)
    yy, xx = np.mgrid[0:H, 0:W].astype(np.float32)
    out = np.empty((T, B, H, W, 2), dtype=np.uint8)
    phase = rng.random(B) * 2 * np.pi
    for t in range(T):
        burst = 0.5 + 0.5 * math.sin(math.pi * t / 40.0) ** 2
        cy = (H / 2 + H / 4 * np.sin(phase + t / 20.0)).astype(np.float32)[:, None, None]
        cx = (W / 2 + W / 4 * np.cos(phase + t / 20.0)).astype(np.float32)[:, None, None]
        blob = np.exp(-((yy - cy) ** 2 + (xx - cx) ** 2) / np.float32(2 * (H / 8) ** 2))
        prob = (0.005 + 0.12 * blob * burst).astype(np.float32)
        u = rng.random((B, H, W, 2), dtype=np.float32)
        out[t] = u < prob[..., None]
    return out


def labels(B: int, classes: int, seed: int = 2) -> np.ndarray:
    return np.random.default_rng(seed).integers(0, classes, size=B).astype(np.int32)


def input_shape(net) -> tuple:
    kind = net["input"]
    if kind[0] == "flat":
        return (kind[1],)
    return (kind[1], kind[2], kind[3])


def make_inputs(net, T: int, B: int, classes: int | None = None, seed: int = 1,
                rate_scale: float = 1.0):
    """(x u8 [T][B][*input], y int32 [B]) for a network."""
    if classes is None:
        classes = net["layers"][-1]["cout"]
    if net["input"][0] == "dvs":
        _, H, W, _c = net["input"]
        x = dvs_frames(T, B, H, W, seed=seed)
    else:
        x = poisson_frames(T, B, input_shape(net), seed=seed, rate_scale=rate_scale)
    y = labels(B, classes, seed=seed + 1)
    return x, y
