"""Pins for the oracle's LIF forward (Eq.1) against closed forms and
hand-worked examples (tests/golden/lif_worked_examples.json)."""
import json
import math
import os

import numpy as np
import pytest

from oracle import lif_step, surrogate_grad
from oracle.bptt import forward_step

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "lif_worked_examples.json")


def run_lif(lam, theta, I, T):
    U = np.zeros(1, np.float32)
    o = np.zeros(1, np.uint8)
    Us, os_ = [], []
    for _ in range(T):
        U, o = lif_step(U, o, np.full(1, I, np.float32), lam, theta)
        Us.append(float(U[0]))
        os_.append(int(o[0]))
    return Us, os_


@pytest.mark.parametrize("case", ["lambda_half", "lambda_one_half_current"])
def test_hand_worked_examples(case):
    g = json.load(open(GOLDEN))[case]
    Us, os_ = run_lif(g["lam"], g["theta"], g["I"], len(g["U"]))
    assert os_ == g["o"]
    assert Us == g["U"]          # dyadic: exact


@pytest.mark.parametrize("I", [0.125, 0.25, 0.375, 0.5, 0.625, 0.75, 0.875, 1.0])
def test_closed_form_integrate_and_fire(I):
    """lam=1, constant dyadic current 0<I<=theta: N_t = ceil((t+1) I/theta) - 1 spikes
    through step t, and U_t = (t+1) I - theta N_{t-1} (unrolled Eq.1 with strict '>')."""
    theta = 1.0
    T = 64
    Us, os_ = run_lif(1.0, theta, I, T)
    N = np.cumsum(os_)
    for t in range(T):
        assert N[t] == math.ceil((t + 1) * I / theta) - 1, t
        Nprev = N[t - 1] if t > 0 else 0
        assert Us[t] == (t + 1) * I - theta * Nprev


@pytest.mark.parametrize("lam,I", [(0.5, 0.75), (0.75, 0.3125), (0.875, 0.25)])
def test_closed_form_leaky_before_first_spike(lam, I):
    """Before the first spike U_t = I (1 - lam^{t+1}) / (1 - lam); first spike at
    min{t : U_t > theta} (geometric series of Eq.1 with o = 0)."""
    theta = 1.0
    T = 30
    Us, os_ = run_lif(lam, theta, I, T)
    closed = [I * (1 - lam ** (t + 1)) / (1 - lam) for t in range(T)]
    first = next((t for t, u in enumerate(closed) if u > theta), None)
    upto = first if first is not None else T - 1
    for t in range(upto + 1):
        assert Us[t] == pytest.approx(closed[t], rel=1e-6)
    if first is None:
        assert sum(os_) == 0
    else:
        assert os_.index(1) == first


def test_network_path_matches_single_neuron():
    """Drive a 1-input fc layer with an all-ones input: the network forward step
    must reproduce the single-neuron worked example."""
    g = json.load(open(GOLDEN))["lambda_half"]
    net = {"input": ("flat", 1), "layers": [
        {"kind": "fc", "cin": 1, "cout": 1, "h": 1, "w": 1, "pool": 0, "lam": g["lam"], "theta": g["theta"]},
        {"kind": "readout", "cin": 1, "cout": 2, "h": 1, "w": 1, "pool": 0, "lam": 1.0, "theta": 0.0}]}
    Wb = [np.array([[g["I"]]]), np.zeros((2, 1))]
    U = [np.zeros((1, 1), np.float32)]
    o = [np.zeros((1, 1), np.uint8)]
    for t in range(len(g["U"])):
        U, o, _ = forward_step(net, Wb, np.ones((1, 1), np.uint8), U, o)
        assert float(U[0][0, 0]) == g["U"][t]
        assert int(o[0][0, 0]) == g["o"][t]


def test_no_fma_order():
    """((lam*U) + I) - theta*o in float32: a case where an FMA would differ."""
    lam, U0, I = np.float32(0.99), np.float32(1.0000001), np.float32(-0.99)
    U, _ = lif_step(np.array([U0]), np.array([0]), np.array([I]), float(lam), 1.0)
    two_roundings = np.float32(np.float32(lam * U0) + I)
    assert U[0] == two_roundings


def test_surrogate_shapes():
    U = np.linspace(-1, 3, 401)
    tri = surrogate_grad(U, 1.0, "triangle", 0.3)
    assert tri.max() == pytest.approx(0.3) and tri[np.argmax(tri)] == tri[200]
    assert np.all(tri[U <= 0] == 0) and np.all(tri[U >= 2] == 0)
    fs = surrogate_grad(U, 1.0, "fast_sigmoid", 2.0)
    assert fs[200] == 1.0 and np.all(fs > 0) and np.all(np.diff(fs[200:]) < 0)
