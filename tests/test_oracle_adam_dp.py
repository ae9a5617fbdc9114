"""Pins: oracle Adam vs torch.optim.Adam (reading 17); data-parallel
linearity with a 2-rank gloo process group (reading 19)."""
import os

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import synth
from oracle import StepConfig, adam_update, train_step


def test_adam_matches_torch():
    rng = np.random.default_rng(0)
    w0 = rng.standard_normal((5, 7))
    p = torch.tensor(w0.copy(), dtype=torch.float64, requires_grad=True)
    opt = torch.optim.Adam([p], lr=1e-3, betas=(0.9, 0.999), eps=1e-8)
    w, m, v = w0.copy(), np.zeros_like(w0), np.zeros_like(w0)
    for step in range(1, 6):
        g = rng.standard_normal(w0.shape) * 10 ** rng.uniform(-4, 1)
        p.grad = torch.tensor(g)
        opt.step()
        w, m, v = adam_update(w, g, m, v, step)
        np.testing.assert_allclose(w, p.detach().numpy(), rtol=1e-14, atol=1e-15)


def test_adam_closed_forms():
    """Closed forms of the bias-corrected update (reading 17): with a constant gradient g the
    corrected moments are exactly g and g^2 at every step, so each step moves w by
    -lr * g / (|g| + eps) (eps = 0: -lr * sign(g)); a zero gradient leaves w and the moments at 0."""
    rng = np.random.default_rng(1)
    w0 = rng.standard_normal(11)
    g = rng.standard_normal(11) * 10 ** rng.uniform(-3, 2, 11)
    lr, eps = 2e-3, 1e-8
    w, m, v = w0.copy(), np.zeros(11), np.zeros(11)
    for step in range(1, 40):
        w, m, v = adam_update(w, g, m, v, step, lr=lr, eps=eps)
        np.testing.assert_allclose(w, w0 - step * lr * g / (np.abs(g) + eps), rtol=1e-12, atol=1e-14)
    w1, _, _ = adam_update(w0, g, np.zeros(11), np.zeros(11), 1, lr=lr, eps=0.0)
    np.testing.assert_allclose(w1, w0 - lr * np.sign(g), rtol=0, atol=1e-15)
    wz, mz, vz = adam_update(w0, np.zeros(11), np.zeros(11), np.zeros(11), 3, lr=lr, eps=eps)
    assert np.array_equal(wz, w0) and not mz.any() and not vz.any()


def _dp_worker(rank, world, port, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    net = synth.net_config("tiny_conv")
    W = synth.make_weights(net)
    T, B = 10, 4
    x, y = synth.make_inputs(net, T, B)
    shard = slice(rank * B // world, (rank + 1) * B // world)
    xs, ys = x[:, shard], y[shard]
    # phase 1: local first pass gives the local s; allreduce it (int64 sum)
    r0 = train_step(net, W, xs, ys, StepConfig(T=T, C=2, mode="ckpt", global_batch=B))
    s = torch.tensor(r0.s)
    dist.all_reduce(s)
    r = train_step(net, W, xs, ys, StepConfig(T=T, C=2, mode="skip", p=50.0, global_batch=B,
                                              s_global=s.numpy()))
    grads = [torch.tensor(g) for g in r.dW]
    for g in grads:
        dist.all_reduce(g)
    loss = torch.tensor([r.loss], dtype=torch.float64)
    dist.all_reduce(loss)
    if rank == 0:
        out.put((float(loss[0]), [g.numpy() for g in grads], r.keep.copy(), s.numpy()))
    dist.destroy_process_group()


def test_data_parallel_sharding_gloo():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29500 + os.getpid() % 1000
    procs = [ctx.Process(target=_dp_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    loss, grads, keep, s = q.get(timeout=300)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    net = synth.net_config("tiny_conv")
    W = synth.make_weights(net)
    x, y = synth.make_inputs(net, 10, 4)
    ref = train_step(net, W, x, y, StepConfig(T=10, C=2, mode="skip", p=50.0))
    np.testing.assert_array_equal(s, ref.s)
    np.testing.assert_array_equal(keep, ref.keep)
    assert loss == pytest.approx(ref.loss, rel=1e-12)
    for a, b in zip(grads, ref.dW):
        np.testing.assert_allclose(a, b, rtol=1e-10, atol=1e-14)


def _dp_bucket_worker(rank, world, port, out):
    """The library's K5 schedule on the host: s allreduced before Eq.5, then dW allreduced in the
    library's layer buckets (flat, top-down), layer 0 and the readout last."""
    from paper_conf_micro_singhslsknnd22_b200 import skipper as sk
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    net = synth.net_config("tiny_resnet")
    W = synth.make_weights(net)
    T, B = 16, 4
    x, y = synth.make_inputs(net, T, B)
    shard = slice(rank * B // world, (rank + 1) * B // world)
    r0 = train_step(net, W, x[:, shard], y[shard], StepConfig(T=T, C=2, mode="ckpt", global_batch=B))
    s = torch.tensor(r0.s)
    dist.all_reduce(s)
    r = train_step(net, W, x[:, shard], y[shard], StepConfig(T=T, C=2, mode="skip", p=50.0, global_batch=B,
                                                             s_global=s.numpy()))
    Ls = len(r.dW) - 1
    nb, closes = sk.plan_buckets([w.size for w in W[:Ls]], 8 << 10)   # small buckets: several of them
    grads = [torch.tensor(g) for g in r.dW]
    hi = Ls - 1
    for i in range(Ls - 1, 0, -1):
        if closes[i]:
            flat = torch.cat([grads[j].flatten() for j in range(i, hi + 1)])
            dist.all_reduce(flat)
            off = 0
            for j in range(i, hi + 1):
                n = grads[j].numel()
                grads[j] = flat[off:off + n].reshape(grads[j].shape)
                off += n
            hi = i - 1
    for j in (0, Ls):
        dist.all_reduce(grads[j])
    if rank == 0:
        out.put((nb, [g.numpy() for g in grads], r.keep.copy()))
    dist.destroy_process_group()


def test_data_parallel_bucketed_allreduce_gloo():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 30500 + os.getpid() % 1000
    procs = [ctx.Process(target=_dp_bucket_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    nb, grads, keep = q.get(timeout=300)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert nb >= 2
    net = synth.net_config("tiny_resnet")
    W = synth.make_weights(net)
    x, y = synth.make_inputs(net, 16, 4)
    ref = train_step(net, W, x, y, StepConfig(T=16, C=2, mode="skip", p=50.0))
    np.testing.assert_array_equal(keep, ref.keep)
    for a, b in zip(grads, ref.dW):
        np.testing.assert_allclose(a, b, rtol=1e-10, atol=1e-14)


def test_batch_slice_pool_equals_full_batch():
    """tests/_oracle_pool.full_batch_train (the full-size backward parity reference): slices with the global
    keep mask and batch size imposed sum to the full-batch oracle step."""
    from _oracle_pool import full_batch_forward, full_batch_train
    from oracle.skipper import keep_mask
    name, T, B, C, p = "tiny_conv", 12, 5, 2, 50.0
    net = synth.net_config(name)
    W = synth.make_weights(net)
    x, y = synth.make_inputs(net, T, B)
    ref = train_step(net, W, x, y, StepConfig(T=T, C=C, p=p, mode="skip"))
    counts, _ = full_batch_forward(name, T, B, C, workers=2)
    np.testing.assert_array_equal(counts, ref.counts)
    keep = keep_mask(counts.sum(axis=0), T, C, p)
    np.testing.assert_array_equal(keep, ref.keep)
    dW, loss = full_batch_train(name, T, B, C, p, "skip", keep, workers=3)
    assert loss == pytest.approx(ref.loss, rel=1e-12)
    for a, b in zip(dW, ref.dW):
        np.testing.assert_allclose(a, b, rtol=1e-12, atol=1e-15)
