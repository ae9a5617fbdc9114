"""Batch-sliced oracle forward passes in worker processes (test helper; samples are independent in the
forward pass of Eq.1, so the first pass of a full-size batch is the concatenation of its slices)."""
import os

for _v in ("OMP_NUM_THREADS", "OPENBLAS_NUM_THREADS", "MKL_NUM_THREADS"):
    os.environ.setdefault(_v, "1")

import numpy as np  # noqa: E402

# results memoised per process: several tests (device variants of one workload) compare against the same
# oracle step
_MEMO = {}


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
    key = ("fwd", name, T, B, C)
    if key in _MEMO:
        return _MEMO[key]
    import concurrent.futures as cf
    import multiprocessing as mp
    workers = workers or max(1, min(len(os.sched_getaffinity(0)), B))
    step = (B + workers - 1) // workers
    jobs = [(name, T, B, C, lo, min(B, lo + step)) for lo in range(0, B, step)]
    with cf.ProcessPoolExecutor(max_workers=len(jobs), mp_context=mp.get_context("spawn")) as ex:
        parts = sorted(ex.map(_slice_forward, jobs), key=lambda r: r[0])
    counts = sum(p[1] for p in parts)
    cnt = np.concatenate([p[2] for p in parts], axis=0)
    _MEMO[key] = (counts, cnt)
    return counts, cnt


def _slice_train(args):
    name, T, B, C, p, mode, keep, lo, hi = args
    import synth
    from oracle import StepConfig, train_step
    net = synth.net_config(name)
    W = synth.make_weights(net)
    x, y = synth.make_inputs(net, T, B)
    exact = mode.endswith("_exact")   # no bf16 rounding of delta (the contract's own effect, deep networks)
    r = train_step(net, W, np.ascontiguousarray(x[:, lo:hi]), y[lo:hi],
                   StepConfig(T=T, C=C, p=p, mode=mode.replace("_exact", ""), keep=keep, global_batch=B,
                              emulate_bf16=not exact))
    return lo, r.dW, r.loss


def full_batch_train(name, T, B, C, p, mode, keep, workers=None):
    """(dW per layer, loss) of the oracle's training step over the whole batch, computed in batch slices:
    every slice runs train_step with the GLOBAL keep mask imposed and the global batch size in the loss
    normalisation, so its weight gradient is the slice's share of the full-batch sum (dW is a sum over
    samples, Eq.2; the cross-entropy is averaged over the global batch, reading 5) - the same
    decomposition the data-parallel mode relies on (reading 19, tests/test_oracle_adam_dp.py)."""
    key = ("train", name, T, B, C, p, mode, None if keep is None else np.asarray(keep).tobytes())
    if key in _MEMO:
        return _MEMO[key]
    import concurrent.futures as cf
    import multiprocessing as mp
    workers = workers or max(1, min(len(os.sched_getaffinity(0)), B))
    step = (B + workers - 1) // workers
    jobs = [(name, T, B, C, p, mode, keep, lo, min(B, lo + step)) for lo in range(0, B, step)]
    with cf.ProcessPoolExecutor(max_workers=len(jobs), mp_context=mp.get_context("spawn")) as ex:
        parts = sorted(ex.map(_slice_train, jobs), key=lambda r: r[0])
    dW = [sum(p_[1][l] for p_ in parts) for l in range(len(parts[0][1]))]
    _MEMO[key] = (dW, sum(p_[2] for p_ in parts))
    return _MEMO[key]
