"""Network topologies and workloads (BASELINE.json `configs`).

A network is a list of layer dicts.  Layers 1..L-1 are spiking LIF layers
(`fc` or `conv` = 3x3, stride 1, pad 1, optional 2x2 average pool of the output
spikes); the last layer is a non-spiking `readout` integrator
(SURVEY.md §8(c) readings 5, 7).  The paper gives only layer counts
(Table I); the channel widths are the proposed ones in
SURVEY.md §8(a).  Activations are NHWC; an `fc` layer after a conv layer reads
the (pooled) conv output flattened in (h, w, c) order.

Per-layer leak lambda and threshold theta are fixed (not trained);
benchmarks use lambda=0.99, theta=1.0 (reading 6).
"""
from __future__ import annotations

import copy

LAM = 0.99
THETA = 1.0


def _conv(cin, cout, hw, pool=0, lam=LAM, theta=THETA, stride=1, res=None):
    """3x3 conv LIF layer; hw = its OUTPUT (neuron) size, the input is hw*stride.
    res = index of the spiking layer whose output spikes enter through the option-A shortcut."""
    d = {"kind": "conv", "cin": cin, "cout": cout, "h": hw, "w": hw,
         "pool": pool, "lam": lam, "theta": theta}
    if stride != 1:
        d["stride"] = stride
    if res is not None:
        d["res"] = res
    return d


def _fc(cin, cout, lam=LAM, theta=THETA):
    return {"kind": "fc", "cin": cin, "cout": cout, "h": 1, "w": 1,
            "pool": 0, "lam": lam, "theta": theta}


def _readout(cin, classes, gap=False):
    d = {"kind": "readout", "cin": cin, "cout": classes, "h": 1, "w": 1,
         "pool": 0, "lam": 1.0, "theta": 0.0}
    if gap:
        d["gap"] = True
    return d


def _resnet(in_hw, in_c, widths, blocks, classes):
    """ResNet-style SNN (SURVEY.md §8(a) cfg 4; Table I "ResNet20"): a stride-2 stem,
    len(widths) stages of `blocks` basic blocks (two 3x3 conv LIF layers; the second one receives the
    block input through the option-A shortcut, reading 8); stages after the first start with a stride-2
    conv; global average pool into the readout (reading 23)."""
    hw = in_hw // 2
    layers = [_conv(in_c, widths[0], hw, stride=2)]
    cin = widths[0]
    for si, wd in enumerate(widths):
        for bi in range(blocks):
            stride = 2 if (si > 0 and bi == 0) else 1
            hw //= stride
            src = len(layers) - 1
            layers.append(_conv(cin, wd, hw, stride=stride))
            layers.append(_conv(wd, wd, hw, res=src))
            cin = wd
    layers.append(_readout(cin, classes, gap=True))
    return layers


def _vgg11(classes=100):
    # [64,A,128,A,256,256,A,512,512,A,512,512,A] on 32x32 (SURVEY.md §8(a) cfg 3)
    return [
        _conv(3, 64, 32, pool=2),
        _conv(64, 128, 16, pool=2),
        _conv(128, 256, 8), _conv(256, 256, 8, pool=2),
        _conv(256, 512, 4), _conv(512, 512, 4, pool=2),
        _conv(512, 512, 2), _conv(512, 512, 2, pool=2),
        _fc(512, 4096), _fc(4096, 4096),
        _readout(4096, classes),
    ]


NETS = {
    # cfg 1: 784-128-10 fully connected (BASELINE.json configs[0])
    "fc784": {"input": ("flat", 784), "layers": [_fc(784, 128), _readout(128, 10)]},
    # cfg 2: VGG-5 style conv(3)+lin(3) (Table I) on CIFAR-10 shape
    "vgg5": {"input": ("image", 32, 32, 3), "layers": [
        _conv(3, 64, 32, pool=2),
        _conv(64, 128, 16),
        _conv(128, 128, 16, pool=2),
        _fc(8192, 1024), _fc(1024, 1024),
        _readout(1024, 10),
    ]},
    # cfg 3 / 5: VGG-11 on CIFAR-100 shape
    "vgg11": {"input": ("image", 32, 32, 3), "layers": _vgg11(100)},
    # small nets for tests (several tiles + ragged tails, all layer kinds)
    "tiny_conv": {"input": ("image", 8, 8, 3), "layers": [
        _conv(3, 64, 8, pool=2),
        _conv(64, 64, 4),
        _conv(64, 128, 4, pool=2),
        _fc(512, 192),
        _readout(192, 10),
    ]},
    "tiny_fc": {"input": ("flat", 40), "layers": [_fc(40, 24), _fc(24, 16), _readout(16, 5)]},
    # cfg 4: ResNet-20-style SNN on DVS-Gesture-shaped event frames (2 x 128 x 128): stem 2-16 s2 -> 64^2,
    # 3 stages x 3 basic blocks (16 @64^2, 32 @32^2, 64 @16^2), GAP -> 11 classes.  19 spiking layers + readout.
    "resnet20_dvs": {"input": ("dvs", 128, 128, 2), "layers": _resnet(128, 2, (16, 32, 64), 3, 11)},
    # small ResNet for tests: both shortcut kinds (identity, stride-2 + channel pad), narrow channels
    "tiny_resnet": {"input": ("dvs", 16, 16, 2), "layers": _resnet(16, 2, (16, 32), 1, 5)},
}


def net_config(name: str, lam: float | None = None, theta: float | None = None):
    """Deep copy of a named topology, optionally overriding lambda/theta of spiking layers."""
    net = copy.deepcopy(NETS[name])
    for layer in net["layers"]:
        if layer["kind"] == "readout":
            continue
        if lam is not None:
            layer["lam"] = float(lam)
        if theta is not None:
            layer["theta"] = float(theta)
    return net


# BASELINE.json configs -> (net, T, B, C, p).  Bold C/p choices of SURVEY.md §8(a).
WORKLOADS = {
    "cfg1_fc784": {"net": "fc784", "T": 20, "B": 4, "C": 2, "p": 50.0, "classes": 10},
    "cfg2_vgg5": {"net": "vgg5", "T": 100, "B": 64, "C": 10, "p": 40.0, "classes": 10},
    "cfg3_vgg11": {"net": "vgg11", "T": 200, "B": 128, "C": 5, "p": 50.0, "classes": 100},
    "cfg4_resnet_dvs": {"net": "resnet20_dvs", "T": 300, "B": 32, "C": 5, "p": 50.0, "classes": 11},
}


def workload(name: str) -> dict:
    return copy.deepcopy(WORKLOADS[name])
