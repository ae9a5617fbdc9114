"""Batch-sliced oracle forward passes in worker processes (test helper; samples are independent in the
forward pass of Eq.1, so the first pass of a full-size batch is the concatenation of its slices)."""
import os

for _v in ("OMP_NUM_THREADS", "OPENBLAS_NUM_THREADS", "MKL_NUM_THREADS"):
    os.environ.setdefault(_v, "1")

import numpy as np  # noqa: E402


def _slice_forward(args):
    name, T, B, C, lo, hi = args
    import synth
    from oracle.bptt import _Ledger, forward_first_pass
    from oracle.numerics import bf16_round
    net = synth.net_config(name)
    W = synth.make_weights(net)
    x, _ = synth.make_inputs(net, T, B)
    Wb = [bf16_round(w) for w in W]
    r = forward_first_pass(net, Wb, x[:, lo:hi], T, T // C, False, _Ledger())
    return lo, r["counts"], r["cnt"]


def full_batch_forward(name, T, B, C, workers=None):
    """(per-layer spike counts [L+1][T] summed over the batch, readout input cnt [B][...]) of the oracle's
    first pass over the whole batch, computed in slices on `workers` processes."""
    import concurrent.futures as cf
    import multiprocessing as mp
    workers = workers or max(1, min(len(os.sched_getaffinity(0)), B))
    step = (B + workers - 1) // workers
    jobs = [(name, T, B, C, lo, min(B, lo + step)) for lo in range(0, B, step)]
    with cf.ProcessPoolExecutor(max_workers=len(jobs), mp_context=mp.get_context("spawn")) as ex:
        parts = sorted(ex.map(_slice_forward, jobs), key=lambda r: r[0])
    counts = sum(p[1] for p in parts)
    cnt = np.concatenate([p[2] for p in parts], axis=0)
    return counts, cnt
