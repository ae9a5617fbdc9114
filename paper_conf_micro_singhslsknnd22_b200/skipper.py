"""Thin ctypes binding of include/skipper.h (argument marshalling only).

Every step of the training path runs in libskipper.so (sm_100a kernels); this
module only converts Python/torch objects into pointers and sizes.  PyTorch is
used for device memory (the caching allocator, so torch's memory statistics
count the library's buffers), streams and process groups.  There is no CPU or
PyTorch fallback: if the library is missing this module raises on import.
"""
from __future__ import annotations

import ctypes as ct
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libskipper.so")

MODE = {"full": 0, "ckpt": 1, "skip": 2, "tbptt": 3}
PASS_FIRST, PASS_RECOMPUTE, PASS_RECORD = 0, 1, 2
LAYER_KIND = {"fc": 0, "conv": 1, "readout": 2}
SURROGATE = {"triangle": 0, "fast_sigmoid": 1}
STATUS = {0: "ok", 1: "EINVAL", 2: "ENOMEM", 3: "ECUDA", 4: "ENCCL", 5: "EORDER", 6: "EFAILED", 7: "EUNSUPPORTED"}


class SkipperError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class Layer(ct.Structure):
    _fields_ = [("kind", ct.c_int), ("cin", ct.c_int), ("cout", ct.c_int), ("h", ct.c_int), ("w", ct.c_int),
                ("pool", ct.c_int), ("lam", ct.c_float), ("theta", ct.c_float), ("stride", ct.c_int),
                ("residual_from", ct.c_int)]


class Config(ct.Structure):
    _fields_ = [("T", ct.c_int), ("C", ct.c_int), ("p", ct.c_double), ("mode", ct.c_int), ("batch", ct.c_int),
                ("global_batch", ct.c_int), ("surrogate", ct.c_int), ("surr_gamma", ct.c_float),
                ("lr", ct.c_float), ("beta1", ct.c_float), ("beta2", ct.c_float), ("eps", ct.c_float),
                ("debug_record", ct.c_int), ("sam", ct.c_int), ("group", ct.c_int)]


ALLOC_FN = ct.CFUNCTYPE(ct.c_void_p, ct.c_size_t, ct.c_void_p, ct.c_void_p)
FREE_FN = ct.CFUNCTYPE(None, ct.c_void_p, ct.c_size_t, ct.c_void_p, ct.c_void_p)


ALLREDUCE_FN = ct.CFUNCTYPE(ct.c_int, ct.c_void_p, ct.c_size_t, ct.c_int, ct.c_void_p, ct.c_void_p)


class _DevArray:
    """__cuda_array_interface__ view of a raw device buffer (torch.as_tensor wraps it without a copy)."""

    def __init__(self, ptr, n, typestr):
        self.__cuda_array_interface__ = {"shape": (int(n),), "typestr": typestr, "data": (int(ptr), False),
                                         "version": 3, "strides": None}


class Allocator(ct.Structure):
    _fields_ = [("alloc", ALLOC_FN), ("free", FREE_FN), ("user", ct.c_void_p)]


def _load():
    # Load torch first so that libskipper.so binds to the same libcudart.so.12 instance as torch
    # (one CUDA runtime per process: shared default-stream semantics, one error state).
    import torch  # noqa: F401
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: run __graft_entry__.build() "
                          "(python -m paper_conf_micro_singhslsknnd22_b200.build)")
    lib = ct.CDLL(LIB_PATH)
    P, I, S = ct.c_void_p, ct.c_int, ct.c_size_t
    sig = {
        "skipper_create": (I, [ct.POINTER(Layer), I, ct.POINTER(Config), ct.POINTER(Allocator), P, ct.POINTER(P)]),
        "skipper_destroy": (None, [P]),
        "skipper_last_error": (ct.c_char_p, [P]),
        "skipper_set_weights": (I, [P, I, P]),
        "skipper_get_weights": (I, [P, I, P]),
        "skipper_get_grads": (I, [P, I, P]),
        "skipper_weight_count": (S, [P, I]),
        "skipper_forward_segment": (I, [P, I, I, P, P]),
        "skipper_backward_segment": (I, [P, I]),
        "skipper_optimizer_step": (I, [P]),
        "skipper_step": (I, [P, P, P, P]),
        "skipper_step_host": (I, [P, P, P, P]),
        "skipper_comm_unique_id": (I, [P]),
        "skipper_comm_init": (I, [P, P, I, I]),
        "skipper_comm_init_callback": (I, [P, ALLREDUCE_FN, P, I, I]),
        "skipper_get_loss": (I, [P, P]),
        "skipper_get_spike_sums": (I, [P, P]),
        "skipper_get_layer_spike_counts": (I, [P, P]),
        "skipper_get_sam": (I, [P, P]),
        "skipper_get_keep_mask": (I, [P, P]),
        "skipper_get_sst": (I, [P, P]),
        "skipper_mem_stats": (I, [P, P, P]),
        "skipper_reset_peak": (I, [P]),
        "skipper_debug_copy": (I, [P, I, I, P, S]),
        "skipper_sst_host": (ct.c_double, [P, I, ct.c_double]),
        "skipper_workspace_bytes": (S, [ct.POINTER(Layer), I, ct.POINTER(Config), I]),
        "skipper_status_string": (ct.c_char_p, [I]),
        "skipper_build_info": (ct.c_char_p, []),
        "skipper_k_fc_fwd": (I, [P, P, P, I, I, I, P]),
        "skipper_k_fc_wgrad": (I, [P, P, P, I, I, I, I, P]),
        "skipper_k_conv_fwd": (I, [P, P, P, I, I, I, I, I, P]),
        "skipper_k_conv_dgrad": (I, [P, P, P, I, I, I, I, I, P]),
        "skipper_k_conv_wgrad": (I, [P, P, P, I, I, I, I, I, I, P]),
        "skipper_k_narrow_wgrad": (I, [P, P, P, I, I, I, I, I, I, I, P]),
        "skipper_k_narrow_dgrad": (I, [P, P, P, I, I, I, I, I, I, P]),
        "skipper_k_conv_lif": (I, [P, P, P, P, P, P, I, I, I, I, I, I, I, ct.c_float, ct.c_float, P]),
        "skipper_k_num_sms": (I, []),
        "skipper_k_conv_s": (I, [P, P, P, I, I, I, I, I, I, I, P]),
        "skipper_k_conv_narrow": (I, [P, P, P, I, I, I, I, I, I, I, P]),
        "skipper_profile": (I, [P, I]),
        "skipper_profile_read": (I, [P, I, P, P, P, P]),
        "skipper_profile_class_name": (ct.c_char_p, [I]),
        "skipper_profile_num_classes": (I, []),
        "skipper_launch_count": (ct.c_longlong, [P]),
        "skipper_profile_records": (ct.c_longlong, [P, P, P, P, P, P, ct.c_longlong]),
        "skipper_plan_buckets": (I, [P, I, ct.c_ulonglong, P]),
        "skipper_encode_poisson": (I, [P, P, ct.c_ulonglong, I, I, ct.c_longlong, P, P]),
        "skipper_step_encoded": (I, [P, P, P, ct.c_ulonglong, P, P]),
        "skipper_step_host_encoded": (I, [P, P, P, ct.c_ulonglong, P, P]),
    }
    for name, (res, args) in sig.items():
        fn = getattr(lib, name)
        fn.restype = res
        fn.argtypes = args
    return lib


lib = _load()


def _check(status, ctx=None):
    if status != 0:
        msg = lib.skipper_last_error(ctx)
        raise SkipperError(status, msg.decode() if msg else "")


def make_layers(net):
    arr = (Layer * len(net["layers"]))()
    for i, L in enumerate(net["layers"]):
        pool = (1 if L.get("gap") else 0) if L["kind"] == "readout" else L.get("pool", 0)
        res = L.get("res")
        arr[i] = Layer(LAYER_KIND[L["kind"]], L["cin"], L["cout"], L.get("h", 1), L.get("w", 1),
                       pool, float(L.get("lam", 1.0)), float(L.get("theta", 1.0)), int(L.get("stride", 1)),
                       -1 if res is None else int(res))
    return arr


SAM = {"spikes": 0, "weighted": 1, "l2trace": 2}


def make_config(T, C=1, p=0.0, mode="skip", batch=1, global_batch=0, surrogate="triangle", gamma=0.3,
                lr=1e-3, beta1=0.9, beta2=0.999, eps=1e-8, debug_record=False, sam="spikes", group=1):
    return Config(T, C, float(p), MODE[mode], batch, global_batch, SURROGATE[surrogate], gamma, lr, beta1, beta2,
                  eps, 1 if debug_record else 0, SAM[sam], int(group))


def sst_host(values, p):
    """Eq.5 for one segment as implemented in the library (host code)."""
    a = np.ascontiguousarray(values, dtype=np.int64)
    return lib.skipper_sst_host(a.ctypes.data, a.size, float(p))


def plan_buckets(wcounts, bucket_bytes):
    """The library's dW-allreduce bucket plan: closes[i] = 1 where a bucket (walking layers n-1 .. 1) ends."""
    wc = np.ascontiguousarray(wcounts, dtype=np.uint64)
    closes = np.zeros(len(wc), dtype=np.int32)
    nb = lib.skipper_plan_buckets(wc.ctypes.data, len(wc), int(bucket_bytes), closes.ctypes.data)
    return nb, closes


def workspace_bytes(net, cfg: Config, kept_max=-1):
    layers = make_layers(net)
    return lib.skipper_workspace_bytes(layers, len(net["layers"]), ct.byref(cfg), kept_max)


def _torch():
    import torch
    return torch


class TorchAllocator:
    """Routes library allocations through torch's CUDA caching allocator."""

    def __init__(self, device):
        torch = _torch()
        self.device = device

        def _alloc(nbytes, stream, user):
            try:
                return torch.cuda.caching_allocator_alloc(int(nbytes), device=self.device, stream=stream or 0)
            except Exception:  # noqa: BLE001 - reported to the library as NULL -> ENOMEM
                return None

        def _free(ptr, nbytes, stream, user):
            if torch is None or getattr(torch, "cuda", None) is None:  # interpreter teardown: memory goes with it
                return
            torch.cuda.caching_allocator_delete(ptr)

        self._a = ALLOC_FN(_alloc)
        self._f = FREE_FN(_free)
        self.struct = Allocator(self._a, self._f, None)


class SkipperNet:
    """One training context (one GPU / rank).  `net` is a synth.configs-style dict."""

    def __init__(self, net, T, C=1, p=0.0, mode="skip", batch=1, global_batch=0, surrogate="triangle",
                 gamma=0.3, lr=1e-3, beta1=0.9, beta2=0.999, eps=1e-8, debug_record=False, stream=None,
                 torch_allocator=True, sam="spikes", group=1):
        torch = _torch()
        self.net = net
        self.T, self.B = T, batch
        self.mode = mode
        self.C = 1 if mode == "full" else C
        self.device = torch.cuda.current_device()
        self.stream = stream if stream is not None else torch.cuda.current_stream()
        self.cfg = make_config(T, C, p, mode, batch, global_batch, surrogate, gamma, lr, beta1, beta2, eps,
                               debug_record, sam, group)
        self._layers = make_layers(net)
        self._alloc = TorchAllocator(self.device) if torch_allocator else None
        h = ct.c_void_p()
        st = _check(lib.skipper_create(self._layers, len(net["layers"]), ct.byref(self.cfg),
                                       ct.byref(self._alloc.struct) if self._alloc else None,
                                       ct.c_void_p(self.stream.cuda_stream), ct.byref(h)))
        del st
        self.ctx = h
        self.n_layers = len(net["layers"])
        self.spiking = [L for L in net["layers"] if L["kind"] != "readout"]

    # ------------------------------------------------------------------ lifecycle
    def close(self):
        if getattr(self, "ctx", None):
            lib.skipper_destroy(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:  # noqa: BLE001
            pass

    def warning(self):
        msg = lib.skipper_last_error(self.ctx)
        return msg.decode() if msg else ""

    def _c(self, status):
        _check(status, self.ctx)

    # ------------------------------------------------------------------ weights
    def weight_count(self, layer):
        return lib.skipper_weight_count(self.ctx, layer)

    def set_weights(self, weights):
        torch = _torch()
        for i, w in enumerate(weights):
            t = torch.as_tensor(np.asarray(w, np.float32) if isinstance(w, np.ndarray) else w)
            t = t.to(device=self.device, dtype=torch.float32).contiguous()
            if t.numel() != self.weight_count(i):
                raise ValueError(f"layer {i}: {t.numel()} weights, expected {self.weight_count(i)}")
            self._c(lib.skipper_set_weights(self.ctx, i, ct.c_void_p(t.data_ptr())))
            self._keep = t
        self.stream.synchronize()

    def _per_layer(self, fn):
        torch = _torch()
        out = []
        for i, L in enumerate(self.net["layers"]):
            shape = (L["cout"], 3, 3, L["cin"]) if L["kind"] == "conv" else (L["cout"], L["cin"])
            t = torch.empty(shape, dtype=torch.float32, device=self.device)
            self._c(fn(self.ctx, i, ct.c_void_p(t.data_ptr())))
            out.append(t)
        self.stream.synchronize()
        return out

    def weights(self):
        return self._per_layer(lib.skipper_get_weights)

    def grads(self):
        return self._per_layer(lib.skipper_get_grads)

    # ------------------------------------------------------------------ training
    def _check_inputs(self, x, y=None):
        torch = _torch()
        if x.dtype != torch.uint8 or not x.is_cuda or not x.is_contiguous() or x.shape[0] != self.T \
                or x.shape[1] != self.B:
            raise ValueError(f"x must be a contiguous CUDA uint8 tensor [T={self.T}][B={self.B}][...]")
        if y is not None and (y.dtype != torch.int32 or not y.is_cuda or y.numel() != self.B):
            raise ValueError(f"labels must be a CUDA int32 tensor of {self.B} elements")

    def step(self, x, y, want_loss=True):
        self._check_inputs(x, y)
        loss = ct.c_float(0.0)
        self._c(lib.skipper_step(self.ctx, ct.c_void_p(x.data_ptr()), ct.c_void_p(y.data_ptr()),
                                 ct.byref(loss) if want_loss else None))
        return float(loss.value) if want_loss else None

    def step_host(self, x_host: np.ndarray, y_host: np.ndarray):
        loss = ct.c_float(0.0)
        self._c(lib.skipper_step_host(self.ctx, ct.c_void_p(x_host.ctypes.data), ct.c_void_p(y_host.ctypes.data),
                                      ct.byref(loss)))
        return float(loss.value)

    def step_encoded(self, x, rates, seed, y, want_loss=True):
        """Poisson-encode x (float32 [B][...] intensities) with rates (float32 [T]) on the device, then step."""
        loss = ct.c_float(0.0)
        self._c(lib.skipper_step_encoded(self.ctx, ct.c_void_p(x.data_ptr()), ct.c_void_p(rates.data_ptr()),
                                         int(seed), ct.c_void_p(y.data_ptr()), ct.byref(loss) if want_loss else None))
        return float(loss.value) if want_loss else None

    def step_host_encoded(self, x_host: np.ndarray, rates_host: np.ndarray, seed: int, y_host: np.ndarray):
        loss = ct.c_float(0.0)
        self._c(lib.skipper_step_host_encoded(self.ctx, ct.c_void_p(x_host.ctypes.data),
                                              ct.c_void_p(rates_host.ctypes.data), int(seed),
                                              ct.c_void_p(y_host.ctypes.data), ct.byref(loss)))
        return float(loss.value)

    def forward_segment(self, seg, pass_, x, y=None):
        self._c(lib.skipper_forward_segment(self.ctx, seg, pass_, ct.c_void_p(x.data_ptr()),
                                            ct.c_void_p(y.data_ptr()) if y is not None else None))

    def backward_segment(self, seg):
        self._c(lib.skipper_backward_segment(self.ctx, seg))

    def optimizer_step(self):
        self._c(lib.skipper_optimizer_step(self.ctx))

    # ------------------------------------------------------------------ data parallel
    @staticmethod
    def comm_unique_id() -> bytes:
        buf = (ct.c_ubyte * 128)()
        _check(lib.skipper_comm_unique_id(buf))
        return bytes(buf)

    def comm_init(self, uid: bytes, rank: int, world: int):
        buf = (ct.c_ubyte * 128).from_buffer_copy(uid)
        self._c(lib.skipper_comm_init(self.ctx, buf, rank, world))

    def comm_init_host(self, rank: int, world: int, group=None):
        """Data parallelism with the collectives on a torch.distributed process group (e.g. gloo) through
        skipper_comm_init_callback: the library issues the same schedule (spike-count allreduce before Eq.5,
        bucketed dW allreduce on its comm stream) and the callback reduces each buffer on the host (stream
        synchronised, device -> host, all_reduce, host -> device).  For several ranks on one GPU, where NCCL
        cannot run; the production path is comm_init (NCCL)."""
        torch = _torch()
        import torch.distributed as dist
        dtypes = {0: (torch.float32, "<f4"), 1: (torch.float64, "<f8"), 2: (torch.int64, "<i8")}

        def _cb(buf, count, dtype, stream, user):
            try:
                if stream:
                    torch.cuda.ExternalStream(stream).synchronize()
                else:
                    torch.cuda.synchronize()
                tdt, ts = dtypes[dtype]
                dev = torch.as_tensor(_DevArray(buf, count, ts), device="cuda")
                host = dev.cpu()
                dist.all_reduce(host, group=group)
                dev.copy_(host)
                torch.cuda.current_stream().synchronize()
                return 0
            except Exception:  # noqa: BLE001 - reported to the library as a failed collective
                import traceback
                traceback.print_exc()
                return 1

        self._allreduce_cb = ALLREDUCE_FN(_cb)   # keep the trampoline alive with the context
        self._c(lib.skipper_comm_init_callback(self.ctx, self._allreduce_cb, None, rank, world))

    # ------------------------------------------------------------------ introspection
    def loss(self):
        v = ct.c_float()
        self._c(lib.skipper_get_loss(self.ctx, ct.byref(v)))
        return float(v.value)

    def spike_sums(self):
        a = np.zeros(self.T, np.int64)
        self._c(lib.skipper_get_spike_sums(self.ctx, a.ctypes.data))
        return a

    def layer_spike_counts(self):
        """[L_n + 1][T] int64 per-layer spike counts of the last first pass (row 0 = input spikes)."""
        a = np.zeros((len(self.spiking) + 1, self.T), np.int64)
        self._c(lib.skipper_get_layer_spike_counts(self.ctx, a.ctypes.data))
        return a

    def sam_values(self):
        """[T] float64: the SAM metric the keep mask was computed from."""
        a = np.zeros(self.T, np.float64)
        self._c(lib.skipper_get_sam(self.ctx, a.ctypes.data))
        return a

    def keep_mask(self):
        a = np.zeros(self.T, np.uint8)
        self._c(lib.skipper_get_keep_mask(self.ctx, a.ctypes.data))
        return a.astype(bool)

    def sst(self):
        a = np.zeros(self.C, np.float64)
        self._c(lib.skipper_get_sst(self.ctx, a.ctypes.data))
        return a

    def mem_stats(self):
        cur, peak = ct.c_size_t(), ct.c_size_t()
        self._c(lib.skipper_mem_stats(self.ctx, ct.byref(cur), ct.byref(peak)))
        return cur.value, peak.value

    def reset_peak(self):
        self._c(lib.skipper_reset_peak(self.ctx))

    def profile(self, enable=True):
        self._c(lib.skipper_profile(self.ctx, 1 if enable else 0))

    def profile_read(self):
        """{class name: dict(launches, ms, bytes, flops)} since the last profile() call (host sync)."""
        out = {}
        for k in range(lib.skipper_profile_num_classes()):
            n, ms, b, f = ct.c_longlong(), ct.c_double(), ct.c_double(), ct.c_double()
            self._c(lib.skipper_profile_read(self.ctx, k, ct.byref(n), ct.byref(ms), ct.byref(b), ct.byref(f)))
            out[lib.skipper_profile_class_name(k).decode()] = {
                "launches": n.value, "ms": ms.value, "bytes": b.value, "flops": f.value}
        return out

    def profile_records(self):
        """Every profiled scope since profile() in launch order: [(class name, kernels, bytes, flops, ms)]."""
        n = lib.skipper_profile_records(self.ctx, None, None, None, None, None, 0)
        if n < 0:
            raise SkipperError(-1, "profile_records on a null context")
        cls = (ct.c_int * n)()
        nk = (ct.c_longlong * n)()
        by = (ct.c_double * n)()
        fl = (ct.c_double * n)()
        ms = (ct.c_float * n)()
        lib.skipper_profile_records(self.ctx, cls, nk, by, fl, ms, n)
        return [(lib.skipper_profile_class_name(cls[i]).decode(), nk[i], by[i], fl[i], ms[i]) for i in range(n)]

    def launch_count(self):
        return lib.skipper_launch_count(self.ctx)

    def debug(self, which, layer):
        """which: 0 first-pass U, 1 first-pass o, 2 recomputed U, 3 recomputed o -> [T][B][neuron shape]."""
        torch = _torch()
        L = self.spiking[layer]
        shape = (L["h"], L["w"], L["cout"]) if L["kind"] == "conv" else (L["cout"],)
        dtype = torch.float32 if which in (0, 2) else torch.uint8
        t = torch.empty((self.T, self.B) + shape, dtype=dtype, device=self.device)
        self._c(lib.skipper_debug_copy(self.ctx, which, layer, ct.c_void_p(t.data_ptr()),
                                       t.numel() * t.element_size()))
        self.stream.synchronize()
        return t


# ---------------------------------------------------------------------- kernel-level entry points
def _ptr(t, dtype=None):
    torch = _torch()
    if not t.is_cuda or not t.is_contiguous():
        raise ValueError("kernel operands must be contiguous CUDA tensors")
    if dtype == "bf16" and t.dtype not in (torch.int16, torch.bfloat16, torch.uint16):
        raise ValueError(f"bf16 operand expected (bf16 or its int16 bit pattern), got {t.dtype}")
    if dtype == "f32" and t.dtype != torch.float32:
        raise ValueError(f"float32 output expected, got {t.dtype}")
    return ct.c_void_p(t.data_ptr())


def _stream_handle():
    return ct.c_void_p(_torch().cuda.current_stream().cuda_stream)


def k_fc_fwd(A, B):
    """C[M][N] = A[M][K] . B[N][K]^T on the tcgen05 path (bf16 in, fp32 out)."""
    torch = _torch()
    M, K = A.shape
    N = B.shape[0]
    out = torch.empty((M, N), dtype=torch.float32, device=A.device)
    _check(lib.skipper_k_fc_fwd(_ptr(A, "bf16"), _ptr(B, "bf16"), _ptr(out, "f32"), M, N, K, _stream_handle()))
    return out


def k_fc_wgrad(D, X, out=None):
    torch = _torch()
    M, N = D.shape
    K = X.shape[1]
    acc = out is not None
    if out is None:
        out = torch.empty((N, K), dtype=torch.float32, device=D.device)
    _check(lib.skipper_k_fc_wgrad(_ptr(D, "bf16"), _ptr(X, "bf16"), _ptr(out, "f32"), M, N, K, 1 if acc else 0, _stream_handle()))
    return out


def k_conv_fwd(X, Wk):
    """X [nb][h][w][cin] bf16, Wk [cout][3][3][cin] bf16 -> Y [nb][h][w][cout] fp32."""
    torch = _torch()
    nb, h, w, cin = X.shape
    cout = Wk.shape[0]
    out = torch.empty((nb, h, w, cout), dtype=torch.float32, device=X.device)
    _check(lib.skipper_k_conv_fwd(_ptr(X, "bf16"), _ptr(Wk, "bf16"), _ptr(out, "f32"), nb, h, w, cin, cout, _stream_handle()))
    return out


def encode_poisson(x, rates, seed):
    """Device Poisson encoder: x float32 [B][D...] (cuda), rates float32 [T] -> uint8 [T][B][D...]."""
    torch = _torch()
    B = x.shape[0]
    D = x[0].numel()
    T = rates.shape[0]
    out = torch.empty((T,) + tuple(x.shape), dtype=torch.uint8, device=x.device)
    _check(lib.skipper_encode_poisson(ct.c_void_p(x.data_ptr()), ct.c_void_p(rates.data_ptr()), int(seed), T, B, D,
                                      ct.c_void_p(out.data_ptr()), _stream_handle()))
    return out


def k_conv_s(X, Wk, stride=1, sign=1, narrow=False):
    """Strided / narrow implicit conv: X [nb][s*h][s*w][cin] bf16, Wk [cout][3][3][cin] bf16 ->
    Y [nb][h][w][cout] fp32 (sign = -1: the stride-1 dgrad form, Wk = Wt).  narrow=True: the cp.async
    gather kernel (skipper_k_conv_narrow) instead of the TMA-box one."""
    torch = _torch()
    nb, hi, wi, cin = X.shape
    cout = Wk.shape[0]
    h, w = hi // stride, wi // stride
    out = torch.empty((nb, h, w, cout), dtype=torch.float32, device=X.device)
    fn = lib.skipper_k_conv_narrow if narrow else lib.skipper_k_conv_s
    _check(fn(_ptr(X, "bf16"), _ptr(Wk, "bf16"), _ptr(out, "f32"), nb, h, w, cin, cout, sign, stride, _stream_handle()))
    return out


def k_conv_lif(X, Wk, U_state, o_state, pool, lam, theta, store_u=True):
    """Fused conv + LIF over R rows.  X [R][nb][h][w][cin] bf16, Wk [cout][3][3][cin] bf16,
    U_state [nb][h][w][cout] fp32 and o_state (uint8) in/out.  Returns (P, U_out): P [R][nb][h'][w'][cout]
    bf16 spikes (2x2 averaged when pool), U_out [R][nb][h][w][cout] fp32 (None unless store_u)."""
    torch = _torch()
    R, nb, h, w, cin = X.shape
    cout = Wk.shape[0]
    if U_state.dtype != torch.float32 or o_state.dtype != torch.uint8:
        raise ValueError("U_state must be float32 and o_state uint8")
    ph, pw = (h // 2, w // 2) if pool else (h, w)
    P = torch.empty((R, nb, ph, pw, cout), dtype=torch.bfloat16, device=X.device)
    U = torch.empty((R, nb, h, w, cout), dtype=torch.float32, device=X.device) if store_u else None
    _check(lib.skipper_k_conv_lif(_ptr(X, "bf16"), _ptr(Wk, "bf16"), _ptr(U_state, "f32"), _ptr(o_state),
                                  _ptr(P, "bf16"), _ptr(U, "f32") if U is not None else None, R, nb, h, w, cin, cout,
                                  1 if pool else 0, float(lam), float(theta), _stream_handle()))
    return P, U


def k_conv_dgrad(D, Wt):
    """D [nb][h][w][cout] bf16, Wt [cin][3][3][cout] bf16 -> G [nb][h][w][cin] fp32."""
    torch = _torch()
    nb, h, w, cout = D.shape
    cin = Wt.shape[0]
    out = torch.empty((nb, h, w, cin), dtype=torch.float32, device=D.device)
    _check(lib.skipper_k_conv_dgrad(_ptr(D, "bf16"), _ptr(Wt, "bf16"), _ptr(out, "f32"), nb, h, w, cin, cout, _stream_handle()))
    return out


def k_narrow_wgrad(D, X, stride=1, out=None):
    """D [nb][h][w][cout], X [nb][stride*h][stride*w][cin] bf16 -> dW [cout][3][3][cin] fp32 (narrow channels)."""
    torch = _torch()
    nb, h, w, cout = D.shape
    cin = X.shape[3]
    acc = out is not None
    if out is None:
        out = torch.empty((cout, 3, 3, cin), dtype=torch.float32, device=D.device)
    _check(lib.skipper_k_narrow_wgrad(_ptr(D, "bf16"), _ptr(X, "bf16"), _ptr(out, "f32"), nb, h, w, cin, cout, stride,
                                      1 if acc else 0, _stream_handle()))
    return out


def k_narrow_dgrad(D, Wt, stride=1):
    """D [nb][h][w][cout], Wt [cin][3][3][cout] bf16 -> G [nb][stride*h][stride*w][cin] fp32 (narrow dgrad)."""
    torch = _torch()
    nb, h, w, cout = D.shape
    cin = Wt.shape[0]
    out = torch.empty((nb, stride * h, stride * w, cin), dtype=torch.float32, device=D.device)
    _check(lib.skipper_k_narrow_dgrad(_ptr(D, "bf16"), _ptr(Wt, "bf16"), _ptr(out, "f32"), nb, h, w, cin, cout, stride,
                                      _stream_handle()))
    return out


def k_conv_wgrad(D, X, out=None):
    """D [nb][h][w][cout], X [nb][h][w][cin] bf16 -> dW [cout][3][3][cin] fp32."""
    torch = _torch()
    nb, h, w, cout = D.shape
    cin = X.shape[3]
    acc = out is not None
    if out is None:
        out = torch.empty((cout, 3, 3, cin), dtype=torch.float32, device=D.device)
    _check(lib.skipper_k_conv_wgrad(_ptr(D, "bf16"), _ptr(X, "bf16"), _ptr(out, "f32"), nb, h, w, cin, cout, 1 if acc else 0,
                                    _stream_handle()))
    return out
