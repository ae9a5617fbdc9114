"""Pins for the oracle's Poisson encoder (NEXT-3): Philox4x32-10 known-answer vectors of
the Random123 distribution, the uniform conversion, and the spike rate law."""
import numpy as np

from oracle.encoder import philox4x32_10, poisson_encode, uniforms

KAT = [  # (counter, key) -> output, philox4x32_10 known-answer tests (Random123 kat_vectors)
    ((0, 0, 0, 0), (0, 0), (0x6627E8D5, 0xE169C58D, 0xBC57AC4C, 0x9B00DBD8)),
    ((0xFFFFFFFF,) * 4, (0xFFFFFFFF, 0xFFFFFFFF), (0x408F276D, 0x41C83B0E, 0xA20BC7C6, 0x6D5451FD)),
    ((0x243F6A88, 0x85A308D3, 0x13198A2E, 0x03707344), (0xA4093822, 0x299F31D0),
     (0xD16CFE09, 0x94FDCCEB, 0x5001E420, 0x24126EA1)),
]


def test_philox_known_answers():
    for ctr, key, out in KAT:
        got = philox4x32_10(*[np.array([c], np.uint64) for c in ctr], *key)
        assert tuple(int(g[0]) for g in got) == out


def test_uniform_conversion_and_range():
    u = uniforms(100003, seed=7)
    assert u.dtype == np.float32 and u.min() >= 0.0 and u.max() < 1.0
    np.testing.assert_array_equal(u * np.float32(2 ** 24), np.floor(u * np.float32(2 ** 24)))
    assert abs(u.mean() - 0.5) < 0.005
    w = philox4x32_10(np.array([0], np.uint64), np.array([0], np.uint64), 0, 0, 7, 0)
    assert u[1] == np.float32((int(w[1][0]) >> 8) * 2.0 ** -24)      # element 1 = word 1 of counter 0


def test_poisson_rate_law():
    rng = np.random.default_rng(0)
    x = rng.random((3, 4000), dtype=np.float32)
    rates = np.array([1.0, 0.5, 0.25, 0.0], np.float32)
    o = poisson_encode(x, rates, seed=3)
    assert o.shape == (4, 3, 4000) and o.dtype == np.uint8
    assert o[3].sum() == 0                                               # zero rate: no spikes
    for t, r in enumerate(rates[:3]):
        assert abs(o[t].mean() - float(r) * float(x.mean())) < 0.01      # E[o] = x r
    assert (poisson_encode(np.ones((1, 10), np.float32), np.ones(1, np.float32), 1) == 1).all()
