"""Pins for SAM / SST / keep mask (Eq.4-5), the checkpoint schedule (Fig. 5/6)
and the memory laws (Eq.3, Eq.6, Eq.7)."""
import json
import math
import os

import numpy as np
import pytest

import synth
from oracle import StepConfig, train_step, keep_mask, spike_sum_threshold, kept_lists
from oracle.skipper import eq7_p_max, ledger_model

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def test_sst_hand_examples():
    for case in json.load(open(os.path.join(GOLD, "sst_hand_examples.json")))["cases"]:
        s = np.array(case["s"])
        keep = keep_mask(s, case["T"], case["C"], case["p"])
        assert keep.astype(int).tolist() == case["keep"], case
        if case["sst"] is not None:
            np.testing.assert_allclose(spike_sum_threshold(s, case["T"], case["C"], case["p"]),
                                       case["sst"], rtol=0, atol=1e-12)


def test_kept_count_order_statistics():
    """With distinct spike sums, exactly S-1-floor((S-1)p/100) values of a segment
    exceed the linear-interpolated percentile (order statistics)."""
    rng = np.random.default_rng(11)
    for _ in range(200):
        C = int(rng.integers(1, 5))
        S = int(rng.integers(2, 30))
        T = C * S
        p = float(rng.uniform(1, 99))
        s = rng.permutation(10 * T)[:T]
        keep = keep_mask(s, T, C, p)
        sst = spike_sum_threshold(s, T, C, p)
        for c in range(C):
            seg = s[c * S:(c + 1) * S]
            n_gt = S - 1 - math.floor((S - 1) * p / 100)
            expect = 1 + n_gt - int(seg[0] > sst[c])
            assert keep[c * S:(c + 1) * S].sum() == expect


def test_sam_brute_force():
    net = synth.net_config("tiny_conv")
    W = synth.make_weights(net)
    T = 10
    x, y = synth.make_inputs(net, T, 3)
    r = train_step(net, W, x, y, StepConfig(T=T, mode="full", record=True))
    for t in range(T):
        brute = int(x[t].astype(np.int64).sum())
        for o in r.first_o:
            brute += int(np.count_nonzero(o[t]))
        assert r.s[t] == brute


def _events(trace, kind):
    return [t for k, t in trace if k == kind]


def test_fig5_schedule_T20_C2():
    g = json.load(open(os.path.join(GOLD, "fig5_schedule_T20_C2.json")))
    net = synth.net_config("tiny_fc")
    W = synth.make_weights(net)
    x, y = synth.make_inputs(net, g["T"], 2)
    r = train_step(net, W, x, y, StepConfig(T=g["T"], C=g["C"], mode="ckpt", trace=True))
    assert _events(r.trace, "ckpt") == g["checkpoints"]
    assert _events(r.trace, "first") == list(range(g["T"]))
    assert _events(r.trace, "loss") == [g["loss_at"]]
    # split the backward part of the trace per release
    seq = r.trace[r.trace.index(("loss", g["loss_at"])) + 1:]
    segs, cur = [], []
    for ev in seq:
        if ev[0] == "release":
            segs.append((ev[1], cur))
            cur = []
        else:
            cur.append(ev)
    assert len(segs) == len(g["segments_in_backward_order"])
    for (c, evs), ref in zip(segs, g["segments_in_backward_order"]):
        assert c == ref["segment"]
        assert _events(evs, "recompute") == ref["recompute"]
        assert _events(evs, "bptt") == ref["bptt"]
    # "the recomputation for each time step happens only once"
    rec = _events(r.trace, "recompute")
    assert len(rec) == len(set(rec)) == g["T"] - g["C"]


def test_fig6_skip_eligibility():
    g = json.load(open(os.path.join(GOLD, "fig5_schedule_T20_C2.json")))
    rng = np.random.default_rng(0)
    for p in [10.0, 50.0, 90.0]:
        s = rng.integers(0, 1000, g["T"])
        keep = keep_mask(s, g["T"], g["C"], p)
        assert keep[0] and keep[10]
        skipped = set(np.nonzero(~keep)[0].tolist())
        assert skipped <= set(sum(g["skipper_eligible"], []))


def test_ledger_matches_eq3_eq6_and_sqrtT():
    net = synth.net_config("tiny_fc")
    W = synth.make_weights(net)
    B = 2
    N = sum(L["cout"] for L in net["layers"] if L["kind"] != "readout")
    T = 36
    x, y = synth.make_inputs(net, T, B)
    per = 5  # U float32 + o uint8 per stored neuron-step
    rf = train_step(net, W, x, y, StepConfig(T=T, mode="full"))
    assert rf.ledger_peak == ledger_model("full", T, 1, per, B * N)
    peaks = {}
    for C in [2, 3, 4, 6, 9, 12, 18]:
        rc = train_step(net, W, x, y, StepConfig(T=T, C=C, mode="ckpt"))
        assert rc.ledger_peak == ledger_model("ckpt", T, C, per, B * N)
        rs = train_step(net, W, x, y, StepConfig(T=T, C=C, mode="skip", p=50.0))
        kmax = max(len(k) for k in rs.kept)
        assert rs.ledger_peak == ledger_model("skip", T, C, per, B * N, kept_max=kmax)
        assert rs.ledger_peak <= rc.ledger_peak < rf.ledger_peak
        peaks[C] = rc.ledger_peak
    assert min(peaks, key=peaks.get) == 6          # C* = sqrt(T)


def test_memory_sublinear_in_T():
    """Eq.3 at C = sqrt(T): ActCost ~ 2 sqrt(T) - quadrupling T doubles memory; FULL is linear."""
    for T in [16, 64, 256]:
        C = int(math.isqrt(T))
        full = ledger_model("full", T, 1, 5, 100)
        ck = ledger_model("ckpt", T, C, 5, 100)
        assert full == T * 500
        assert ck == 2 * C * 500
    assert ledger_model("ckpt", 256, 16, 5, 1) / ledger_model("ckpt", 64, 8, 5, 1) == 2


def test_eq7_bounds_for_workloads():
    assert eq7_p_max(100, 10, 6) == pytest.approx(40.0)    # cfg 2 -> p=40
    assert eq7_p_max(200, 5, 11) == pytest.approx(72.5)    # cfg 3
    assert eq7_p_max(20, 2, 2) == pytest.approx(80.0)      # cfg 1


# ---------------------------------------------------------------- NEXT-2: neuron-count-weighted SAM
def test_sam_weighted_hand_example():
    """Reading 22 on a hand-worked case: counts [[2,0,4],[1,3,0]], neurons [2, 4]."""
    from oracle.skipper import sam_weighted
    s = sam_weighted(np.array([[2, 0, 4], [1, 3, 0]]), [2, 4])
    assert s.tolist() == [1.25, 0.75, 2.0]


def test_sam_weighted_equal_sizes_reduces_to_spike_sum():
    """With every layer the same (power-of-two) size the weighted metric is the spike sum / N, and the
    percentile threshold and keep mask are scale-equivariant: the masks are identical."""
    from oracle.skipper import sam_weighted
    rng = np.random.default_rng(3)
    for _ in range(200):
        T, C = 40, 4
        counts = rng.integers(0, 300, size=(3, T))
        p = float(rng.choice([10, 25, 40, 50, 75]))
        w = sam_weighted(counts, [64, 64, 64])
        assert np.array_equal(keep_mask(w, T, C, p), keep_mask(counts.sum(0), T, C, p))


def test_sam_weighted_network_brute_force():
    """train_step(sam='weighted'): the policy metric equals the per-layer firing counts recorded in the
    first pass divided by the layer sizes, and the mask is the Eq.5 rule applied to it."""
    net = synth.net_config("tiny_conv")
    W = synth.make_weights(net, seed=0)
    x, y = synth.make_inputs(net, 12, 3, seed=1)
    res = train_step(net, W, x, y, StepConfig(T=12, C=2, p=50.0, mode="skip", sam="weighted", record=True))
    n0 = int(np.prod(x.shape[2:]))
    brute = np.array([x[t].astype(np.int64).sum() / n0 +
                      sum(res.first_o[l][t].astype(np.int64).sum() / res.first_o[l][t][0].size
                          for l in range(len(res.first_o))) for t in range(12)])
    assert np.allclose(res.sam, brute, rtol=1e-15, atol=0)
    assert np.array_equal(res.keep, keep_mask(res.sam, 12, 2, 50.0))
    assert res.counts.shape == (len(res.first_o) + 1, 12)
    assert np.array_equal(res.counts.sum(0), res.s)


def test_sam_weighted_changes_the_mask_somewhere():
    """The variant is live: on the VGG-5 topology (layers of very different sizes) the weighted and
    plain metrics select different steps for some seed."""
    net = synth.net_config("tiny_conv")
    W = synth.make_weights(net, seed=0)
    differ = False
    for seed in range(1, 8):
        x, y = synth.make_inputs(net, 20, 2, seed=seed)
        a = train_step(net, W, x, y, StepConfig(T=20, C=2, p=50.0, mode="skip"))
        b = train_step(net, W, x, y, StepConfig(T=20, C=2, p=50.0, mode="skip", sam="weighted"))
        differ |= not np.array_equal(a.keep, b.keep)
        if differ:
            break
    assert differ


def test_l2trace_sam_brute_force_and_mask():
    """NEXT-2 second variant (reading 25): s_t = ||U_t||_2 over every spiking neuron of the
    first pass; recomputed here from the recorded membranes, and the mask is the Eq.5 rule applied to it."""
    import synth
    from oracle import StepConfig, train_step
    net = synth.net_config("tiny_conv")
    W = synth.make_weights(net)
    T, C, p = 20, 2, 50.0
    x, y = synth.make_inputs(net, T, 3)
    r = train_step(net, W, x, y, StepConfig(T=T, C=C, p=p, mode="skip", sam="l2trace", record=True))
    brute = np.zeros(T)
    for t in range(T):
        tot = 0.0
        for U in r.first_U:
            for v in np.asarray(U[t], np.float64).ravel():
                tot += v * v
        brute[t] = np.sqrt(tot)
    np.testing.assert_allclose(r.sam, brute, rtol=1e-13)
    S = T // C
    for c in range(C):
        seg = brute[c * S:(c + 1) * S]
        thr = np.percentile(seg, p)
        keep = seg > thr
        keep[0] = True
        np.testing.assert_array_equal(r.keep[c * S:(c + 1) * S], keep)
    assert 0 < r.keep.sum() < T
