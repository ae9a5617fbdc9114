"""Diagnostic: per-layer dW error of the device against the batch-sliced oracle at a given workload size.
usage: python tools/diag_grad.py NAME T B C p [ENV=VAL ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402


def main():
    name, T, B, C, p = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4]), float(sys.argv[5])
    for kv in sys.argv[6:]:
        k, v = kv.split("=")
        os.environ[k] = v
    from _oracle_pool import full_batch_forward, full_batch_train
    from oracle.skipper import keep_mask
    from paper_conf_micro_singhslsknnd22_b200 import SkipperNet
    net = synth.net_config(name)
    W = synth.make_weights(net)
    x, y = synth.make_inputs(net, T, B)
    m = SkipperNet(net, T, C=C, p=p, mode="skip", batch=B)
    m.set_weights(W)
    loss = m.step(torch.from_numpy(x).cuda(), torch.from_numpy(y).cuda())
    grads = [g.cpu().numpy().astype(np.float64) for g in m.grads()]
    counts, _ = full_batch_forward(name, T, B, C)
    keep = keep_mask(counts.sum(axis=0), T, C, p)
    assert np.array_equal(m.keep_mask(), keep)
    dW, ref_loss = full_batch_train(name, T, B, C, p, "skip", keep)
    print(f"{name} T={T} B={B} C={C} p={p} {sys.argv[6:]} loss {loss:.6f} ref {ref_loss:.6f}")
    for l, (g, r) in enumerate(zip(grads, dW)):
        nw = np.linalg.norm(g - r) / max(np.linalg.norm(r), 1e-30)
        mx = np.abs(g - r).max() / max(np.abs(r).max(), 1e-30)
        ratio = np.linalg.norm(g) / max(np.linalg.norm(r), 1e-30)
        print(f"  layer {l}: normwise {nw:.2e} maxabs {mx:.2e} |g|/|r| {ratio:.6f}")


if __name__ == "__main__":
    main()
