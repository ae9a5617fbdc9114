"""Full, checkpointed and Skipper BPTT training steps - test infrastructure only.

PAPER.md citations (P:<line>):
* baseline BPTT stores every (U, o) and back-propagates once (Fig. 1a/2);
* checkpointing (Sec. V, Fig. 5): the first forward saves the state
  only at t = cS; for c = C-1..0 the segment is recomputed from its checkpoint
  "only once", back-propagated, and its memory released;
  the error gradient at the segment start is carried to the previous segment
  (Step 3 / Step 5);
* Skipper (Sec. VI-A, Fig. 6): the first forward also records s_t
  (Eq.4); before recomputing segment c, SST_c (Eq.5) decides which t are kept;
  "a shallower computation graph" over the kept steps only is built and
  back-propagated.  Reading A:
  kept steps chain directly, U_{k_j} = lam U_{k_{j-1}} + W o^{l-1}_{k_j} - theta o_{k_{j-1}},
  and the delta after the last kept step of segment c is the carry from c+1.
* Eq.2: delta^l_t = sigma'(U^l_t) * (W^{l+1 T} delta^{l+1}_t) + lam * delta^l_{t+1},
  dW^l = sum_t delta^l_t (o^{l-1}_t)^T, reset detached.

Readout and loss (reading 5, "loss ... at t=19"): non-spiking
integrator z = (1/T) W^L sum_t a^{L-1}_t, softmax cross-entropy summed over the
local batch and divided by the global batch.  Readout gradients run over the
kept steps only (reading 15).  A readout marked "gap" integrates the global
average pool of a^{L-1} (the ResNet20 SNN, reading 23).

ResNet layers (reading 8): a conv layer may have stride 2 (its h, w are the
output = neuron dims) and a residual source "res" = index r of an earlier
spiking layer: the option-A shortcut of a^r is added into the layer's current,
I = W * a^{l-1} + S(a^r) (exact sum, rounded once to float32), and Eq.2's
gradient wrt a^r gains S^T(delta^l).

Arithmetic contract: forward currents are the exact
sum of bf16 weights times spike inputs, rounded once to float32 (exact for the
grid weights of the parity tests); LIF in float32 (oracle/lif.py); backward in
float64 with bf16 rounding of delta before the dgrad/wgrad contractions.
dW accumulates per layer in descending t, so CKPT reproduces FULL bit for bit.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

from .layers import (conv3x3, conv3x3_input_grad, conv3x3_weight_grad, gap, gap_T, pool2, pool2_T,
                     shortcut_a, shortcut_a_T)
from .lif import lif_step, surrogate_grad
from .numerics import bf16_round
from .skipper import keep_mask, kept_lists, sam_weighted, spike_sum_threshold


@dataclass
class StepConfig:
    T: int
    C: int = 1
    p: float = 0.0
    mode: str = "full"            # "full" | "ckpt" | "skip" | "tbptt"
    surrogate: str = "triangle"
    gamma: float = 0.3
    global_batch: int | None = None
    emulate_bf16: bool = True     # round delta to bf16 at the GEMM inputs
    keep: np.ndarray | None = None       # test hook: impose a keep mask (skip mode)
    dz: np.ndarray | None = None         # test hook: impose the readout gradient
    T_norm: int | None = None            # readout normalisation (default T)
    s_global: np.ndarray | None = None   # data-parallel: allreduced s (reading 19)
    sam: str = "spikes"                  # SAM metric: "spikes" (Eq.4) | "weighted" (reading 22) | "l2trace" (reading 25)
    counts_global: np.ndarray | None = None  # data-parallel: allreduced per-layer counts (weighted SAM)
    u2_global: np.ndarray | None = None      # data-parallel: allreduced sum of U^2 per t (l2-trace SAM)
    record: bool = False
    trace: bool = False


@dataclass
class StepResult:
    loss: float
    z: np.ndarray
    dz: np.ndarray
    s: np.ndarray                 # int64 [T], local batch
    counts: np.ndarray            # int64 [L_n + 1][T] per-layer spike counts (row 0 = input), local batch
    sam: np.ndarray               # the policy metric the mask is computed from (int64 or float64 [T])
    sst: np.ndarray | None        # float64 [C] (skip mode)
    keep: np.ndarray              # bool [T]
    kept: list                    # per segment, ascending kept t
    dW: list                      # float64 per layer (spiking layers, then readout)
    cnt: np.ndarray               # readout input summed over all T (first pass)
    cnt_kept: np.ndarray          # readout input summed over kept t
    ledger_peak: int              # stored-state bytes at the peak (Eq.3 / Eq.6)
    first_U: list = field(default_factory=list)   # [l] float32 [T][B][...]
    first_o: list = field(default_factory=list)   # [l] uint8   [T][B][...]
    rec_U: list = field(default_factory=list)     # [l] float32 [T][B][...], kept t only
    rec_o: list = field(default_factory=list)
    trace: list = field(default_factory=list)


def spiking_layers(net):
    return [L for L in net["layers"] if L["kind"] != "readout"]


def neuron_shape(layer) -> tuple:
    if layer["kind"] == "conv":
        return (layer["h"], layer["w"], layer["cout"])
    return (layer["cout"],)


def out_shape(layer) -> tuple:
    if layer["kind"] == "conv" and layer["pool"]:
        return (layer["h"] // 2, layer["w"] // 2, layer["cout"])
    return neuron_shape(layer)


def synaptic_current(layer, Wb, a_in, a_res=None) -> np.ndarray:
    """I = W^l P(o^{l-1}) (Eq.1 second term) [+ S(a^r), reading 8]: exact float64 sum, rounded once to float32."""
    B = a_in.shape[0]
    if layer["kind"] == "conv":
        I = conv3x3(a_in, Wb, layer.get("stride", 1))
        if a_res is not None:
            I = I + shortcut_a(a_res, a_res.shape[1] // layer["h"], layer["cout"])
    else:
        I = a_in.reshape(B, -1) @ Wb.T
    return I.astype(np.float32)


def layer_output(layer, o) -> np.ndarray:
    """a^l = P(o^l): the value the next layer integrates (reading 7)."""
    if layer["kind"] == "conv" and layer["pool"]:
        return pool2(o)
    return np.asarray(o, np.float64)


def forward_step(net, Wb, x_t, U_prev, o_prev):
    """Eq.1 through every spiking layer at one timestep.

    Returns (U list, o list, a list) with a[0] = input spikes, a[l+1] = P(o^l)."""
    a = [np.asarray(x_t, np.float64)]
    Us, os_ = [], []
    for l, layer in enumerate(spiking_layers(net)):
        r = layer.get("res")
        I = synaptic_current(layer, Wb[l], a[l], None if r is None else a[r + 1])
        U, o = lif_step(U_prev[l], o_prev[l], I, layer["lam"], layer["theta"])
        Us.append(U)
        os_.append(o)
        a.append(layer_output(layer, o))
    return Us, os_, a


def spike_sum(x_t, os_) -> int:
    """Eq.4 at one t: input spikes plus every spiking layer's spikes (reading 11)."""
    return int(np.asarray(x_t, np.int64).sum()) + sum(int(np.asarray(o, np.int64).sum()) for o in os_)


def readout_input(cnt, use_gap: bool) -> np.ndarray:
    """What the readout integrates: the summed a^{L-1}, flattened, or its global average pool (reading 23)."""
    return gap(cnt) if use_gap else np.asarray(cnt, np.float64).reshape(cnt.shape[0], -1)


def readout(WbL, cnt, y, T_norm: int, B_global: int, use_gap: bool = False):
    """z = W^L cnt / T; loss = sum_b CE(z_b, y_b) / B_global; dz = (softmax - onehot) / B_global."""
    B = cnt.shape[0]
    c2 = readout_input(cnt, use_gap)
    z = c2 @ WbL.T / T_norm
    zmax = z.max(axis=1, keepdims=True)
    e = np.exp(z - zmax)
    lse = np.log(e.sum(axis=1)) + zmax[:, 0]
    loss = float((lse - z[np.arange(B), y]).sum() / B_global)
    prob = e / e.sum(axis=1, keepdims=True)
    onehot = np.zeros_like(prob)
    onehot[np.arange(B), y] = 1.0
    dz = (prob - onehot) / B_global
    return loss, z, dz


class _Ledger:
    """Bytes of stored neuron state (U float32 + o uint8 = 5 B / neuron / stored step)."""

    def __init__(self):
        self.live = 0
        self.peak = 0

    def add(self, arrays):
        self.live += sum(int(a.nbytes) for a in arrays)
        self.peak = max(self.peak, self.live)

    def sub(self, arrays):
        self.live -= sum(int(a.nbytes) for a in arrays)


def forward_first_pass(net, Wb, x, T: int, S: int, store_all: bool, ledger: _Ledger,
                       record: bool = False, trace=None):
    """First forward pass (Fig. 5 / Fig. 6 Step 1).

    store_all (FULL / RECORD): keep (U, o, a) of every t.  Otherwise keep only
    the state after step cS (the checkpoint) for every segment.  Always records
    s_t (SAM) and the readout input summed over t."""
    spk = spiking_layers(net)
    B = x.shape[1]
    U = [np.zeros((B,) + neuron_shape(L), np.float32) for L in spk]
    o = [np.zeros((B,) + neuron_shape(L), np.uint8) for L in spk]
    s = np.zeros(T, np.int64)
    counts = np.zeros((len(spk) + 1, T), np.int64)
    u2 = np.zeros(T, np.float64)          # sum over every spiking neuron of U_t^2 (l2-trace SAM, reading 25)
    cnt = np.zeros((B,) + out_shape(spk[-1]), np.float64)
    ckpt = {}
    stored = []          # FULL: list over t of (U list, o list, a list)
    first_U = [np.zeros((T,) + u.shape, np.float32) for u in U] if record else []
    first_o = [np.zeros((T,) + u.shape, np.uint8) for u in U] if record else []
    for t in range(T):
        U, o, a = forward_step(net, Wb, x[t], U, o)
        s[t] = spike_sum(x[t], o)
        counts[0, t] = int(np.asarray(x[t], np.int64).sum())
        for l in range(len(spk)):
            counts[l + 1, t] = int(np.asarray(o[l], np.int64).sum())
            u2[t] += float(np.sum(np.asarray(U[l], np.float64) ** 2))
        cnt += a[-1]
        if record:
            for l in range(len(spk)):
                first_U[l][t] = U[l]
                first_o[l][t] = o[l]
        if store_all:
            stored.append((U, o, a))
            ledger.add(U + o)
        elif t % S == 0:
            ckpt[t // S] = ([u.copy() for u in U], [v.copy() for v in o])
            ledger.add(ckpt[t // S][0] + ckpt[t // S][1])
            if trace is not None:
                trace.append(("ckpt", t))
        if trace is not None:
            trace.append(("first", t))
    return {"s": s, "counts": counts, "u2": u2, "cnt": cnt, "ckpt": ckpt, "stored": stored,
            "first_U": first_U, "first_o": first_o}


def recompute_segment(net, Wb, x, ckpt_c, rows, ledger: _Ledger, trace=None):
    """Second forward over the kept rows of one segment (Fig. 5 Step 2/4, Fig. 6 Step 2).

    Row 0 (t = cS) is the checkpoint itself; rows j >= 1 chain from row j-1
    (reading A).  Returns per-row (U list, o list, a list)."""
    spk = spiking_layers(net)
    U0, o0 = ckpt_c
    a0 = [np.asarray(x[rows[0]], np.float64)] + [layer_output(L, o0[l]) for l, L in enumerate(spk)]
    out = [(U0, o0, a0)]
    ledger.add(U0 + o0)            # the segment's stored row 0 (aliases the checkpoint values)
    U, o = U0, o0
    for t in rows[1:]:
        U, o, a = forward_step(net, Wb, x[t], U, o)
        out.append((U, o, a))
        ledger.add(U + o)
        if trace is not None:
            trace.append(("recompute", int(t)))
    return out


def backward_segment(net, Wb, rows_state, dz, T_norm, carry, dW, cnt_kept, cfg: StepConfig,
                     rows=None, trace=None):
    """BPTT over one (possibly compacted) segment, Eq.2, float64.

    rows_state: per row ascending in t, (U list, o list, a list).
    carry[l]: delta^l at the first row of the next segment (zero for the last).
    Returns the new carry (delta^l at this segment's row 0)."""
    spk = spiking_layers(net)
    Ls = len(spk)
    K = len(rows_state)
    B = dz.shape[0]
    WbL = Wb[Ls]
    use_gap = bool(net["layers"][-1].get("gap"))
    # readout input summed over the kept rows (readout gradients over kept t, reading 15)
    for j in reversed(range(K)):
        cnt_kept += rows_state[j][2][Ls]
    # grad wrt the readout input, identical at every kept t: dz W^L / T (through the GAP when present)
    ga_const = dz @ WbL / T_norm
    if use_gap:
        ga_const = gap_T(ga_const, out_shape(spk[-1])[:2])
    ga_const = ga_const.reshape((B,) + out_shape(spk[-1]))
    ga = [ga_const] * K
    ga_res = {}                                                   # residual source r -> S^T(delta) per row
    new_carry = [None] * Ls
    for l in reversed(range(Ls)):
        layer = spk[l]
        lam = float(layer["lam"])
        pooled = layer["kind"] == "conv" and layer["pool"]
        if l in ga_res:                                           # dL/da^l also flows through the shortcut
            extra = ga_res.pop(l)
            ga = [ga[j] + extra[j] for j in range(K)]
        g = [pool2_T(gj) if pooled else gj for gj in ga]           # dL/do^l_t (spatial path)
        delta = [None] * K
        nxt = carry[l]
        for j in reversed(range(K)):
            sg = surrogate_grad(rows_state[j][0][l], layer["theta"], cfg.surrogate, cfg.gamma)
            delta[j] = sg * g[j] + lam * nxt                      # Eq.2
            nxt = delta[j]
        new_carry[l] = delta[0]
        db = [bf16_round(d) for d in delta] if cfg.emulate_bf16 else delta
        stride = layer.get("stride", 1)
        for j in reversed(range(K)):                              # dW^l += delta_t^T a^{l-1}_t
            a_in = rows_state[j][2][l]
            if layer["kind"] == "conv":
                dW[l] += conv3x3_weight_grad(db[j], a_in, stride)
            else:
                dW[l] += db[j].reshape(B, -1).T @ a_in.reshape(B, -1)
        r = layer.get("res")
        if r is not None:                                          # S^T delta^l into dL/da^r
            a_r = rows_state[0][2][r + 1]
            prev = ga_res.get(r, [0.0] * K)
            ga_res[r] = [prev[j] + shortcut_a_T(db[j], a_r.shape[1] // layer["h"], a_r.shape[3], a_r.shape[1:3])
                         for j in range(K)]
        if l > 0:                                                  # grad wrt a^{l-1}: W^{l T} delta^l
            a_shape = rows_state[0][2][l].shape
            if layer["kind"] == "conv":
                ga = [conv3x3_input_grad(db[j], Wb[l], stride, a_shape[1:3]) for j in range(K)]
            else:
                ga = [(db[j].reshape(B, -1) @ Wb[l]).reshape(a_shape) for j in range(K)]
    if trace is not None and rows is not None:
        for t in reversed(list(rows)):
            trace.append(("bptt", int(t)))
    return new_carry


def tbptt_step(net, W, x, y, cfg: StepConfig) -> StepResult:
    """Truncated BPTT (Sec. III-C), NEXT-4 of SURVEY.md §8(f).

    The network is unrolled over truncation windows of t' = T/C steps.  At the end of window w a loss
    is computed from the readout integrated over that window, z_w = W^L (sum_{t in w} a^{L-1}_t) / t'
    (reading 24), its derivatives are back-propagated through the window only (the graph of earlier
    windows is discarded: delta after the window's last step is zero), and the weight gradients of all
    windows are summed.  The neuron state (U, o) itself carries on across windows.  The
    reported loss is the sum of the window losses, so the gradient is the (truncated) gradient of it."""
    spk = spiking_layers(net)
    Ls = len(spk)
    T, C = cfg.T, cfg.C
    if T % C:
        raise ValueError("C must divide T")
    S = T // C
    B = x.shape[1]
    B_global = cfg.global_batch or B
    use_gap = bool(net["layers"][-1].get("gap"))
    Wb = [bf16_round(w) for w in W]
    ledger = _Ledger()
    U = [np.zeros((B,) + neuron_shape(L), np.float32) for L in spk]
    o = [np.zeros((B,) + neuron_shape(L), np.uint8) for L in spk]
    s = np.zeros(T, np.int64)
    counts = np.zeros((Ls + 1, T), np.int64)
    dW = [np.zeros(w.shape, np.float64) for w in W]
    loss_tot = 0.0
    first_U = [np.zeros((T, B) + neuron_shape(L), np.float32) for L in spk] if cfg.record else []
    first_o = [np.zeros((T, B) + neuron_shape(L), np.uint8) for L in spk] if cfg.record else []
    cnt_all = np.zeros((B,) + out_shape(spk[-1]), np.float64)
    z = dz = None
    for w in range(C):
        rows_state = []
        cnt = np.zeros((B,) + out_shape(spk[-1]), np.float64)
        for t in range(w * S, (w + 1) * S):
            U, o, a = forward_step(net, Wb, x[t], U, o)
            s[t] = spike_sum(x[t], o)
            counts[0, t] = int(np.asarray(x[t], np.int64).sum())
            for l in range(Ls):
                counts[l + 1, t] = int(np.asarray(o[l], np.int64).sum())
                if cfg.record:
                    first_U[l][t] = U[l]
                    first_o[l][t] = o[l]
            cnt += a[-1]
            rows_state.append((U, o, a))
            ledger.add(U + o)
        cnt_all += cnt
        loss_w, z, dz = readout(Wb[Ls], cnt, y, S, B_global, use_gap)
        loss_tot += loss_w
        carry = [np.zeros((B,) + neuron_shape(L), np.float64) for L in spk]     # the graph is cut here
        cnt_w = np.zeros_like(cnt)
        backward_segment(net, Wb, rows_state, dz, S, carry, dW, cnt_w, cfg)
        dW[Ls] += dz.T @ readout_input(cnt_w, use_gap) / S
        for st in rows_state:                     # the window's graph is released
            ledger.sub(st[0] + st[1])
    keep = np.ones(T, bool)
    return StepResult(loss=loss_tot, z=z, dz=dz, s=s, counts=counts, sam=s, sst=None, keep=keep,
                      kept=kept_lists(keep, T, C), dW=dW, cnt=cnt_all, cnt_kept=cnt_all, ledger_peak=ledger.peak,
                      first_U=first_U, first_o=first_o, rec_U=first_U, rec_o=first_o)


def train_step(net, W, x, y, cfg: StepConfig) -> StepResult:
    """One training iteration's gradients (no optimizer step; see oracle/adam.py).

    W: float32 master weights per layer (spiking layers then readout).
    x: uint8 [T][B][...] input spikes, y: int [B] labels."""
    if cfg.mode == "tbptt":
        return tbptt_step(net, W, x, y, cfg)
    spk = spiking_layers(net)
    Ls = len(spk)
    T = cfg.T
    B = x.shape[1]
    B_global = cfg.global_batch or B
    T_norm = cfg.T_norm or T
    mode = cfg.mode
    C = 1 if mode == "full" else cfg.C
    if T % C:
        raise ValueError("C must divide T (P:1779-1781)")
    S = T // C
    Wb = [bf16_round(w) for w in W]
    ledger = _Ledger()
    trace = [] if cfg.trace else None

    first = forward_first_pass(net, Wb, x, T, S, store_all=(mode == "full"), ledger=ledger,
                               record=cfg.record, trace=trace)
    s = first["s"]
    use_gap = bool(net["layers"][-1].get("gap"))
    loss, z, dz = readout(Wb[Ls], first["cnt"], y, T_norm, B_global, use_gap)
    if trace is not None:
        trace.append(("loss", T - 1))
    if cfg.dz is not None:
        dz = np.asarray(cfg.dz, np.float64)

    if cfg.sam == "weighted":
        counts = first["counts"] if cfg.counts_global is None else np.asarray(cfg.counts_global, np.int64)
        neurons = [int(np.prod(x.shape[2:]))] + [int(np.prod(neuron_shape(L))) for L in spk]
        s_pol = sam_weighted(counts, neurons)
    elif cfg.sam == "l2trace":
        u2 = first["u2"] if cfg.u2_global is None else np.asarray(cfg.u2_global, np.float64)
        s_pol = np.sqrt(u2)
    elif cfg.sam == "spikes":
        s_pol = s if cfg.s_global is None else np.asarray(cfg.s_global, np.int64)
    else:
        raise ValueError(f"unknown SAM metric {cfg.sam!r}")
    sst = None
    if mode == "skip":
        if cfg.keep is not None:
            keep = np.asarray(cfg.keep, bool).copy()
        else:
            keep = keep_mask(s_pol, T, C, cfg.p)
            if cfg.p != 0:
                sst = spike_sum_threshold(s_pol, T, C, cfg.p)
    else:
        keep = np.ones(T, bool)
    kept = kept_lists(keep, T, C)

    dW = [np.zeros(w.shape, np.float64) for w in W]
    cnt_kept = np.zeros_like(first["cnt"])
    carry = [np.zeros((B,) + neuron_shape(L), np.float64) for L in spk]
    rec_U = [np.zeros((T, B) + neuron_shape(L), np.float32) for L in spk] if cfg.record else []
    rec_o = [np.zeros((T, B) + neuron_shape(L), np.uint8) for L in spk] if cfg.record else []

    if mode == "full":
        rows_state = first["stored"]
        carry = backward_segment(net, Wb, rows_state, dz, T_norm, carry, dW, cnt_kept, cfg,
                                 rows=range(T), trace=trace)
        if cfg.record:
            for t in range(T):
                for l in range(Ls):
                    rec_U[l][t] = rows_state[t][0][l]
                    rec_o[l][t] = rows_state[t][1][l]
    else:
        for c in reversed(range(C)):
            rows = kept[c]
            rows_state = recompute_segment(net, Wb, x, first["ckpt"][c], rows, ledger, trace)
            carry = backward_segment(net, Wb, rows_state, dz, T_norm, carry, dW, cnt_kept, cfg,
                                     rows=rows, trace=trace)
            if cfg.record:
                for j, t in enumerate(rows):
                    for l in range(Ls):
                        rec_U[l][t] = rows_state[j][0][l]
                        rec_o[l][t] = rows_state[j][1][l]
            for st in rows_state:                 # release the segment
                ledger.sub(st[0] + st[1])
            if trace is not None:
                trace.append(("release", c))
    # readout weight gradient once, over the kept rows of every segment
    dW[Ls] += dz.T @ readout_input(cnt_kept, use_gap) / T_norm
    return StepResult(loss=loss, z=z, dz=dz, s=s, counts=first["counts"], sam=s_pol, sst=sst, keep=keep, kept=kept, dW=dW,
                      cnt=first["cnt"], cnt_kept=cnt_kept, ledger_peak=ledger.peak,
                      first_U=first["first_U"], first_o=first["first_o"],
                      rec_U=rec_U, rec_o=rec_o, trace=trace or [])
