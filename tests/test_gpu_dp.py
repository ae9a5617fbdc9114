"""K5 (the data-parallel regime of P:676-682) on the device with TWO ranks.

Two processes share the one GPU of the test box (NCCL cannot put two ranks on one device), each training its
half of the batch through the C ABI; the collectives of the library's data-parallel schedule - the int64
per-layer spike counts before Eq.5 and the bucketed fp32 dW allreduce issued on the comm stream during
segment 0's backward - go through skipper_comm_init_callback to a gloo process group.  The ranks' keep masks,
summed loss and weight gradients must equal the oracle's full-batch step (reading 19: the global s gives the
single-GPU mask; dW is a sum over samples) and a one-process device step on the whole batch."""
import os
import tempfile

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import synth
from oracle import StepConfig, train_step

pytestmark = pytest.mark.gpu


def _rank(rank, world, port, name, T, B, C, p, out, bucket_mb):
    os.environ.update({"MASTER_ADDR": "127.0.0.1", "MASTER_PORT": str(port), "SKIPPER_BUCKET_MB": str(bucket_mb)})
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    from paper_conf_micro_singhslsknnd22_b200 import SkipperNet
    net = synth.net_config(name)
    W = synth.make_weights(net)
    x, y = synth.make_inputs(net, T, B)
    h = B // world
    xs = np.ascontiguousarray(x[:, rank * h:(rank + 1) * h])
    ys = np.ascontiguousarray(y[rank * h:(rank + 1) * h])
    m = SkipperNet(net, T, C=C, p=p, mode="skip", batch=h, global_batch=B)
    m.set_weights(W)
    m.comm_init_host(rank, world)
    loss = m.step(torch.from_numpy(xs).cuda(), torch.from_numpy(ys).cuda())
    res = {"loss": np.array([loss]), "keep": m.keep_mask(), "s": m.spike_sums()}
    for l, g in enumerate(m.grads()):
        res[f"g{l}"] = g.cpu().numpy()
    for l, w in enumerate(m.weights()):
        res[f"w{l}"] = w.cpu().numpy()
    np.savez(os.path.join(out, f"rank{rank}.npz"), **res)
    m.close()
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("name,T,B,C,p,bucket_mb", [("tiny_conv", 12, 4, 2, 50.0, 1), ("vgg5", 14, 4, 2, 40.0, 1),
                                                    ("tiny_resnet", 16, 4, 2, 50.0, 1), ("fc784", 20, 4, 2, 50.0, 25)])
def test_two_rank_device_data_parallel(name, T, B, C, p, bucket_mb):
    from paper_conf_micro_singhslsknnd22_b200 import SkipperNet
    world = 2
    port = 29600 + (abs(hash((name, T, B))) % 300)
    with tempfile.TemporaryDirectory() as out:
        mp.start_processes(_rank, args=(world, port, name, T, B, C, p, out, bucket_mb), nprocs=world, join=True,
                           start_method="spawn")
        ranks = [dict(np.load(os.path.join(out, f"rank{r}.npz"))) for r in range(world)]
    net = synth.net_config(name)
    W = synth.make_weights(net)
    x, y = synth.make_inputs(net, T, B)
    ref = train_step(net, W, x, y, StepConfig(T=T, C=C, p=p, mode="skip"))
    # one-process device step on the whole batch
    m = SkipperNet(net, T, C=C, p=p, mode="skip", batch=B)
    m.set_weights(W)
    loss1 = m.step(torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda())
    g1 = [g.cpu().numpy() for g in m.grads()]
    m.close()
    for r in ranks:   # the allreduced s gives every rank the full-batch mask (reading 19)
        np.testing.assert_array_equal(r["s"], ref.s)
        np.testing.assert_array_equal(r["keep"], ref.keep)
    assert sum(float(r["loss"][0]) for r in ranks) == pytest.approx(ref.loss, rel=1e-5)
    assert sum(float(r["loss"][0]) for r in ranks) == pytest.approx(loss1, rel=1e-5)
    for l, dref in enumerate(ref.dW):
        a, b = ranks[0][f"g{l}"].astype(np.float64), ranks[1][f"g{l}"].astype(np.float64)
        np.testing.assert_array_equal(a, b)                # allreduced: identical on both ranks
        np.testing.assert_array_equal(ranks[0][f"w{l}"], ranks[1][f"w{l}"])   # same Adam step
        if np.linalg.norm(dref) == 0:
            assert np.abs(a).max() == 0
            continue
        assert np.linalg.norm(a - dref) <= 1e-3 * np.linalg.norm(dref), l
        assert np.abs(a - dref).max() <= 1e-3 * np.abs(dref).max(), l
        assert np.linalg.norm(a - g1[l]) <= 1e-5 * np.linalg.norm(g1[l]) + 1e-12, l
