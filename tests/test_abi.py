"""CPU-side checks of the C ABI boundary: the library loads, exports every symbol
the headers declare, and its host logic (Eq.5 SST, validation of P:840-853 /
P:1779-1781, the Eq.3/Eq.6 storage model) behaves - no GPU needed."""
import ctypes
import os
import re

import numpy as np
import pytest

import synth
from paper_conf_micro_singhslsknnd22_b200 import skipper as sk

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    names = set()
    for h in ["skipper.h", "skipper_kernels.h"]:
        src = open(os.path.join(ROOT, "include", h)).read()
        src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
        names |= set(re.findall(r"\b(skipper_[a-z0-9_]+)\s*\(", src))
    return sorted(names)


def test_all_declared_symbols_exported():
    names = declared_functions()
    assert len(names) > 30
    lib = ctypes.CDLL(sk.LIB_PATH)
    missing = [n for n in names if not hasattr(lib, n)]
    assert not missing, missing


def test_library_is_sm100a():
    data = open(sk.LIB_PATH, "rb").read()
    assert b"sm_100a" in data


def test_sst_host_matches_numpy_percentile():
    rng = np.random.default_rng(0)
    for _ in range(3000):
        n = int(rng.integers(1, 40))
        hi = int(rng.choice([3, 20, 10 ** 6]))
        s = rng.integers(0, hi, n)
        p = float(rng.choice([rng.uniform(0, 100), 10.0, 25.0, 33.3, 40.0, 50.0, 52.0, 70.0, 90.0, 99.9]))
        assert sk.sst_host(s, p) == np.percentile(s, p), (s, p)


def test_sst_host_hand_cases():
    assert sk.sst_host([5, 3, 8, 1, 9, 2, 7, 4, 6, 0], 50.0) == 4.5
    assert sk.sst_host([1, 9, 2, 8], 25.0) == 1.75


def _create(net, **cfg):
    layers = sk.make_layers(net)
    c = sk.make_config(**cfg)
    h = ctypes.c_void_p()
    st = sk.lib.skipper_create(layers, len(net["layers"]), ctypes.byref(c), None, None, ctypes.byref(h))
    return st, sk.lib.skipper_last_error(None).decode()


@pytest.mark.parametrize("cfg,needle", [
    (dict(T=20, C=3, p=50.0, mode="skip", batch=2), "divide"),
    (dict(T=20, C=10, p=50.0, mode="skip", batch=2), "exceed"),
    (dict(T=20, C=2, p=100.0, mode="skip", batch=2), "outside"),
    (dict(T=20, C=2, p=-1.0, mode="ckpt", batch=2), "outside"),
    (dict(T=0, C=1, p=0.0, mode="full", batch=2), "positive"),
])
def test_create_rejects_invalid_config(cfg, needle):
    st, msg = _create(synth.net_config("fc784"), **cfg)
    assert st == 1 and needle in msg, msg


def test_create_rejects_bad_topology():
    net = synth.net_config("vgg5")
    net["layers"][3]["cin"] = 4096
    st, msg = _create(net, T=20, C=2, p=0.0, mode="ckpt", batch=2)
    assert st == 1 and "cin" in msg
    net = synth.net_config("fc784")
    net["layers"] = net["layers"][:-1]
    st, msg = _create(net, T=20, C=2, p=0.0, mode="ckpt", batch=2)
    assert st == 1 and "readout" in msg


def test_workspace_model_laws():
    """Eq.3: FULL linear in T; CKPT minimal near C = sqrt(T); Eq.6: SKIP below CKPT."""
    net = synth.net_config("vgg5")
    full = [sk.workspace_bytes(net, sk.make_config(T=T, mode="full", batch=8)) for T in (100, 200, 400)]
    assert full[1] == 2 * full[0] and full[2] == 4 * full[0]
    T = 400
    ck = {C: sk.workspace_bytes(net, sk.make_config(T=T, C=C, mode="ckpt", batch=8)) for C in (4, 10, 16, 20, 25, 40, 50)}
    best = min(ck, key=ck.get)
    assert best in (16, 20, 25)
    sk40 = sk.workspace_bytes(net, sk.make_config(T=T, C=20, p=50.0, mode="skip", batch=8), kept_max=11)
    assert sk40 < ck[20] < full[2]


def test_status_strings_and_build_info():
    assert sk.lib.skipper_status_string(0) == b"ok"
    assert sk.lib.skipper_status_string(5) == b"call order violation"
    assert b"sm_100a" in sk.lib.skipper_build_info()


def buckets_from_plan(closes):
    """Layer ranges [lo, hi] of the buckets, in the order the library launches them (top layer first)."""
    out, hi = [], len(closes) - 1
    for i in range(len(closes) - 1, 0, -1):
        if closes[i]:
            out.append((i, hi))
            hi = i - 1
    return out


@pytest.mark.parametrize("name", ["vgg5", "vgg11", "resnet20_dvs", "fc784", "tiny_fc"])
@pytest.mark.parametrize("mb", [1, 25, 1000])
def test_bucket_plan_partitions_layers(name, mb):
    """K5 bucket plan: every spiking layer >= 1 in exactly one contiguous bucket, each
    bucket but the last at least bucket_bytes, launched top-down (the order segment 0 finalises dW)."""
    net = synth.net_config(name)
    spk = [L for L in net["layers"] if L["kind"] != "readout"]
    from synth.inputs import weight_shape
    wc = [int(np.prod(weight_shape(L))) for L in spk]
    nb, closes = sk.plan_buckets(wc, mb << 20)
    if len(spk) == 1:
        assert nb == 0 and not closes.any()
        return
    b = buckets_from_plan(closes)
    assert nb == len(b) and b[-1][0] == 1 and b[0][1] == len(spk) - 1
    covered = sorted(i for lo, hi in b for i in range(lo, hi + 1))
    assert covered == list(range(1, len(spk)))
    for lo, hi in b[:-1]:
        assert 4 * sum(wc[lo:hi + 1]) >= mb << 20
        assert 4 * sum(wc[lo + 1:hi + 1]) < mb << 20      # closed as soon as it was full


def test_workspace_model_tbptt():
    """TBPTT stores one truncation window: T/C steps of U + outputs, independent of T at fixed t'."""
    net = synth.net_config("vgg5")
    full = sk.workspace_bytes(net, sk.make_config(T=100, mode="full", batch=8))
    tb = [sk.workspace_bytes(net, sk.make_config(T=T, C=T // 10, mode="tbptt", batch=8)) for T in (100, 400)]
    assert tb[0] == tb[1] == full // 10


def test_tbptt_validation():
    net = synth.net_config("tiny_fc")
    st, msg = _create(net, T=12, C=5, mode="tbptt", batch=2)
    assert st == 1 and "divide" in msg
    st, _ = _create(net, T=12, C=12, mode="tbptt", batch=2)   # t' = 1 is a valid truncation window
    assert st == 0 or st == 3   # 3 = no CUDA device on the CPU box
