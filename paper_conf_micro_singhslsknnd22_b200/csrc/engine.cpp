// engine.cpp - the C ABI of include/skipper.h: context, validation, memory plan and the
// segment schedule of checkpointed / Skipper BPTT (Sec. V Fig. 5, Sec. VI-A Fig. 6).
//
// Per iteration (SKIP mode):
//   stage input (SAM l=0) -> FIRST pass over segments 0..C-1 (layer-major inside a segment:
//   GEMM over all S timesteps, then the LIF scan walks t; checkpoint (U,o) at t=cS) ->
//   readout + loss -> [allreduce s] -> host SST_c (Eq.5) and keep lists (one host sync) ->
//   for c = C-1..0 { RECOMPUTE kept rows from checkpoint c ; BACKWARD: K4 scan, wgrad, dgrad }
//   -> [allreduce dW] -> Adam.
#include "../../include/skipper.h"
#include "gemm.h"
#include "kernels.h"

#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <string>
#include <unordered_map>
#include <vector>

#include "comm.h"

namespace {

thread_local std::string g_last_error;

struct Layer {
    skipper_layer d{};
    bool fc = false, conv = false, pool = false, readout = false;
    int H = 1, W = 1, Cin = 0, Cout = 0, PH = 1, PW = 1;
    int stride = 1, Hin = 1, Win = 1;  // conv: output (neuron) H x W, input (stride H) x (stride W)
    int res = -1, res_to = -1;          // ResNet: residual source layer (this = receiver) / receiver (this = source)
    bool icol = false;                  // conv via explicit im2col + GEMM (narrow / strided layers)
    bool fwd_s = false, dgrad_s = false;  // icol layer whose forward / dgrad runs as the narrow implicit conv
    bool fwd_g = false, dgrad_g = false;  // ... through the cp.async gather kernel (conv_narrow.cu)
    bool nlif = false;                    // gather conv + LIF scan fused (conv_narrow.cu, LIF epilogue)
    bool gap = false;                   // readout integrates the global average pool (reading 23)
    long long N = 0, Nout = 0, Nin = 0;  // per sample: neurons, outputs (after pool), inputs
    size_t wcount = 0;
    float *w = nullptr, *dw = nullptr, *m = nullptr, *v = nullptr;
    uint16_t *wb = nullptr, *wt = nullptr;
    float *U_run = nullptr, *ckU = nullptr, *carry = nullptr;
    uint8_t *o_run = nullptr, *cko = nullptr;
    uint16_t *Po = nullptr;    // arena rows
    uint16_t *PoS[2] = {nullptr, nullptr};  // the two slots of Po (ctx.wdb)
    float *Useg = nullptr;     // arena rows
    int fsplit = 1, dsplit = 1;  // split-K factors of the forward / dgrad GEMMs (fc layers, fixed per layer)
    int fsplitT = 1;             // forward split-K of the chunked first pass (fc tail layers, tail_G*S rows)
    bool cfused = false;         // conv layer: GEMM + LIF scan as one kernel (conv_lif.cu)
    bool dlif = false;           // this layer's dgrad runs with layer i-1's reverse scan in its epilogue
                                 // (conv_lif.cu BWD, NEXT-1 backward half): g^{i-1} never reaches HBM
    size_t sbn = 0;              // elements of one running-state / checkpoint slot (B*N, or conv_lif's
                                 // thread-major layout, conv_lif_state_count, when cfused)
    // deterministic split-K weight gradient: wsl > 0 -> the wgrad launches add into slice s of dws
    // [wsl][wg_count] (one writer per slice per launch), summed in slice order into dW (or dwp) after the
    // layer's last weight-gradient launch of the step (launch_reduce_slices)
    float *dws = nullptr;
    int wsl = 0;
    bool wsl_narrow = false;   // the slices are narrow_wgrad's per-CTA partials
    size_t wg_count = 0;
    uint16_t *wbp = nullptr;   // layer 0 im2col: bf16 weights zero-padded to [cout][K0]
    float *dwp = nullptr;      // layer 0 im2col: padded weight gradient
    float *dbg[2] = {nullptr, nullptr};     // first / recompute U
    uint8_t *dbgo[2] = {nullptr, nullptr};  // first / recompute o
};

enum Phase { PH_IDLE = 0, PH_FIRST, PH_READY_BWD, PH_RECOMPUTED, PH_BWD_DONE };

// GEMM plans (three encoded TMA descriptors each) are cached by operand pointers and shape: the
// segment arenas come back at the same addresses step after step, so steady-state steps encode no
// tensor maps on the host.
struct PlanKey {
    int op;
    const void *a, *b;
    const void *c;
    long long M;
    int N, K, h, w, x;
    bool operator==(const PlanKey &o) const {
        return op == o.op && a == o.a && b == o.b && c == o.c && M == o.M && N == o.N && K == o.K && h == o.h &&
               w == o.w && x == o.x;
    }
};
struct PlanKeyHash {
    size_t operator()(const PlanKey &k) const {
        size_t h = std::hash<const void *>()(k.a);
        auto mix = [&h](size_t v) { h ^= v + 0x9e3779b97f4a7c15ULL + (h << 6) + (h >> 2); };
        mix(std::hash<const void *>()(k.b));
        mix(std::hash<const void *>()(k.c));
        mix((size_t)k.M);
        mix((size_t)k.op * 131 + k.N);
        mix((size_t)k.K * 31 + k.h * 7 + k.w * 3 + k.x);
        return h;
    }
};

}  // namespace

struct skipper_ctx {
    std::vector<Layer> L;  // spiking layers then readout (L.back())
    int Ls = 0;            // number of spiking layers
    skipper_config cfg{};
    skipper_allocator alloc{};
    bool own_alloc = true;
    cudaStream_t st = nullptr;
    // side stream: the weight-gradient GEMM of layer l runs there, overlapping the dgrad of layer l
    // and the reverse scan of layer l-1 on the main stream (delta is double-buffered)
    cudaStream_t st2 = nullptr;
    cudaEvent_t ev_ready[3] = {nullptr, nullptr, nullptr}, ev_done[3] = {nullptr, nullptr, nullptr};
    bool w_pending[3] = {false, false, false};
    // weight gradients across segment borders (per-segment SKIP / CKPT schedule): the layer outputs and the
    // layer-0 operand rows - the weight gradients' X operands - alternate between two arena slots by
    // segment parity, so segment c's weight gradients run on under the recompute of c-1 instead of being
    // joined before it (the slot is waited for only when segment c-2 reuses it)
    bool wdb = false;
    int cur_slot = 0;
    cudaEvent_t ev_slot[2] = {nullptr, nullptr};
    bool slot_rec[2] = {false, false};
    int T = 0, C = 1, S = 0, B = 0, Bg = 0;
    int num_sms = 148;
    int in_kind = 0;            // layer-0 operand: 0 fc rows, 1 3x3 im2col rows (K0 cols), 2 NHWC image
    int K0 = 0;                 // im2col width (32 or 64)
    bool l0_fused = false;      // layer 0 runs as the fused im2col+tcgen05+LIF kernel (layer0.cu)
    bool l0_bwd_fused = false;  // layer 0 backward: fused reverse scan + tcgen05 weight gradient
    int tail0 = 0;              // first layer of the fc tail: the first pass runs it per chunk of tail_G segments
    int F = 1;                  // segments per first-pass launch of the layers before the fc tail
    int fp_s0 = 0;              // first segment of the first-pass chunk in progress
    int tail_G = 1;             // segments per fc-tail chunk (tail_G * S * B <= max(SKIPPER_TAIL_ROWS, S * B) rows,
                                // independent of T: keeps Eq.3's O(C) + O(S) law)
    uint16_t *tail_in = nullptr, *tailP[2] = {nullptr, nullptr};
    float *tail_I = nullptr;
    int in_h = 1, in_w = 1, in_c = 0;
    long long in_elems = 0;     // input elements per sample (uint8 x)
    long long in_row = 0;       // staged bf16 layer-0 operand elements per sample
    // persistent
    unsigned *s_part = nullptr;
    double *u2_part = nullptr, *u2_dev = nullptr;  // l2-trace SAM: [T][32] partials, [T] totals
    std::vector<double> u2_host;
    long long *s_dev = nullptr;
    float *cnt = nullptr, *cnt_kept = nullptr, *z = nullptr, *dz = nullptr, *loss_dev = nullptr, *g_last = nullptr;
    int *kept_dev = nullptr;
    float *dw_all = nullptr;
    size_t dw_total = 0;
    unsigned char *x_stage = nullptr;
    int *y_stage = nullptr;
    unsigned char *x_enc = nullptr;                           // on-device encoded spikes [T][B][D]
    float *img_stage = nullptr, *rates_stage = nullptr;       // host-encoded path staging
    // host-side step state
    std::vector<long long> s_host;         // Eq.4 spike sums [T]
    std::vector<long long> counts_host;    // per-layer spike counts [(Ls + 1)][T], row 0 = input
    std::vector<double> sam_host;          // the SAM metric thresholded by Eq.5 [T]
    std::vector<unsigned char> keep;
    std::vector<double> sst;
    std::vector<std::vector<int>> kept;
    std::vector<int> kept_flat;
    int Kmax = 0;
    // backward groups (skipper_config.group = G): segments c_lo..c_lo+G-1 are recomputed one at a time into
    // consecutive rows of one arena (ascending time) and back-propagated as ONE layer-major pass over the
    // concatenated kept rows (the carry rule of Eq.2 across the segment border is the reverse scan's own)
    int G = 1;
    std::vector<int> seg_lo, seg_off, grp_R, grp_start;  // per segment: its group's lowest segment, row offset;
                                                         // per lowest segment: group rows, start in grp_dev
    std::vector<int> grp_flat;
    int *grp_dev = nullptr;
    int Rgrp = 0;                                        // arena rows: max over groups of the kept rows
    // arenas
    void *arena = nullptr;
    size_t arena_bytes = 0;
    float *I_buf = nullptr;     // currents (fwd) and gradients wrt spikes (dgrad)
    uint16_t *d_buf = nullptr;  // delta (bf16)
    uint16_t *d_buf2[3] = {nullptr, nullptr, nullptr};  // delta ring (3 deep when residuals exist)
    uint16_t *P2[3] = {nullptr, nullptr, nullptr};      // FIRST-pass output ring (3 deep when residuals exist)
    int nD = 2, nP = 2;
    uint16_t *cols[3] = {nullptr, nullptr, nullptr};    // im2col operands of icol layers (per delta slot)
    float *dcols = nullptr;                             // icol dgrad output columns (fp32)
    float *cnt_gap = nullptr, *g_gap = nullptr;         // GAP readout input / gradient [B][C]
    uint16_t *xg = nullptr;     // staged layer-0 operand rows of the current pass
    uint16_t *xgS[2] = {nullptr, nullptr};  // the two slots of xg (wdb)
    // schedule state
    int phase = PH_IDLE;
    int next_seg = 0;
    bool grads_ready = false;
    long long adam_step = 0;
    const unsigned char *x_cur = nullptr;
    // memory accounting
    size_t cur_bytes = 0, peak_bytes = 0;
    std::string err;
    bool poisoned = false;
    // comm: one NCCL communicator (K5).  The dW allreduce runs in layer buckets on st3 while segment 0's
    // backward continues (a bucket of layers hi..lo is final once lo's weight gradient has run in
    // segment 0); layer 0 (unpadded at the end) and the readout follow on the same stream.
    sk::Comm comm;
    cudaStream_t st3 = nullptr;
    cudaEvent_t ev_w = nullptr, ev_comm = nullptr;
    std::vector<int> bucket_lo;   // per spiking layer i >= 1: 1 if layer i closes a bucket
    bool comm_pending = false;
    std::unordered_map<PlanKey, sk::GemmLaunch, PlanKeyHash> plans;
    // profiling (per kernel class: launches, device ms, algorithmic bytes and flops)
    bool prof_on = false;
    std::vector<cudaEvent_t> ev_pool;
    size_t ev_used = 0;
    struct ProfRec { int cls; cudaEvent_t a, b; double bytes, flops; long long k0, nk; };
    std::vector<ProfRec> prof_recs;
    struct ProfLog { int cls; long long nk; double bytes, flops; float ms; };
    std::vector<ProfLog> prof_log;   // every profiled scope in launch order (ncu attribution, tools/ncu_classes.py)
    long long prof_n[16] = {0};
    double prof_ms[16] = {0}, prof_bytes[16] = {0}, prof_flops[16] = {0};
    long long launches = 0;
    // host-side phase timing (SKIPPER_HOST_PROFILE=1, printed at destroy): issue of the first pass, the
    // mask sync wait, issue of recompute + backward + optimizer
    bool host_prof = false;
    double hp_first = 0, hp_sync = 0, hp_bwd = 0, hp_gap = 0;
    cudaEvent_t hp_ev[2] = {nullptr, nullptr};  // device timeline: the mask D2H done / the first RECOMPUTE work
    long long hp_steps = 0;
};

static double now_ms() {
    return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

enum KClass {
    K_STAGE = 0, K_GEMM_FWD, K_SCAN_FWD, K_READOUT, K_SCAN_BWD, K_GEMM_WGRAD, K_GEMM_DGRAD, K_ADAM, K_UNPAD,
    K_L0_FWD, K_L0_BWD, K_CONV_LIF, K_IM2COL, K_DGRAD_LIF, K_NCLASS
};
static const char *k_class_names[K_NCLASS] = {"stage_input", "gemm_fwd", "lif_fwd_scan", "readout_loss",
                                               "lif_bwd_scan", "gemm_wgrad", "gemm_dgrad", "adam", "unpad",
                                               "layer0_fused_fwd", "layer0_fused_bwd", "gemm_lif_fwd", "im2col",
                                               "gemm_lif_bwd"};

static cudaEvent_t ev_get(skipper_ctx *c) {
    if (c->ev_used < c->ev_pool.size()) return c->ev_pool[c->ev_used++];
    cudaEvent_t e;
    cudaEventCreate(&e);
    c->ev_pool.push_back(e);
    c->ev_used++;
    return e;
}

// One kernel launch: counts it and, when profiling, brackets it with CUDA events on the
// context stream together with its algorithmic bytes / flops.
struct ProfScope {
    skipper_ctx *c;
    cudaStream_t s;
    int rec = -1;
    ProfScope(skipper_ctx *c_, int cls, double bytes, double flops, cudaStream_t s_ = nullptr) : c(c_), s(s_) {
        if (!s) s = c->st;
        const long long k0 = c->launches++;
        if (!c->prof_on) return;
        cudaEvent_t a = ev_get(c), b = ev_get(c);
        cudaEventRecord(a, s);
        c->prof_recs.push_back({cls, a, b, bytes, flops, k0, 1});
        rec = (int)c->prof_recs.size() - 1;
    }
    ~ProfScope() {
        if (rec < 0) return;
        cudaEventRecord(c->prof_recs[rec].b, s);
        c->prof_recs[rec].nk = c->launches - c->prof_recs[rec].k0;  // kernels launched inside the scope
    }
};

static void prof_resolve(skipper_ctx *c) {
    if (c->prof_recs.empty()) return;
    for (auto &r : c->prof_recs) cudaEventSynchronize(r.b);
    for (auto &r : c->prof_recs) {
        float ms = 0.f;
        if (cudaEventElapsedTime(&ms, r.a, r.b) == cudaSuccess) {
            c->prof_n[r.cls] += 1;
            c->prof_ms[r.cls] += ms;
            c->prof_bytes[r.cls] += r.bytes;
            c->prof_flops[r.cls] += r.flops;
        }
        c->prof_log.push_back({r.cls, r.nk, r.bytes, r.flops, ms});
    }
    c->prof_recs.clear();
    c->ev_used = 0;
}

// ------------------------------------------------------------------------------------ helpers
static skipper_status fail(skipper_ctx *c, skipper_status s, const char *fmt, ...) {
    char buf[1024];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    if (c) {
        c->err = buf;
        if (s == SKIPPER_ECUDA || s == SKIPPER_ENCCL) c->poisoned = true;
    }
    g_last_error = buf;
    return s;
}

#define CK(call)                                                                                     \
    do {                                                                                             \
        cudaError_t e_ = (call);                                                                     \
        if (e_ != cudaSuccess)                                                                       \
            return fail(c, SKIPPER_ECUDA, "%s:%d %s: %s", __FILE__, __LINE__, #call, cudaGetErrorString(e_)); \
    } while (0)

#define CKS(expr)                            \
    do {                                     \
        skipper_status s_ = (expr);          \
        if (s_ != SKIPPER_OK) return s_;     \
    } while (0)

static size_t al256(size_t n) { return (n + 255) & ~size_t(255); }

static void *dev_alloc(skipper_ctx *c, size_t bytes) {
    if (bytes == 0) return nullptr;
    bytes = al256(bytes);
    void *p = nullptr;
    if (c->own_alloc) {
        if (cudaMallocAsync(&p, bytes, c->st) != cudaSuccess) p = nullptr;
    } else {
        p = c->alloc.alloc(bytes, c->st, c->alloc.user);
    }
    if (p) {
        c->cur_bytes += bytes;
        c->peak_bytes = std::max(c->peak_bytes, c->cur_bytes);
    }
    return p;
}

static void dev_free(skipper_ctx *c, void *p, size_t bytes) {
    if (!p) return;
    bytes = al256(bytes);
    if (c->own_alloc)
        cudaFreeAsync(p, c->st);
    else
        c->alloc.free(p, bytes, c->st, c->alloc.user);
    c->cur_bytes -= bytes;
}

template <typename T>
static skipper_status alloc_arr(skipper_ctx *c, T **p, size_t n) {
    *p = static_cast<T *>(dev_alloc(c, n * sizeof(T)));
    if (n && !*p) return fail(c, SKIPPER_ENOMEM, "device allocation of %zu bytes failed", n * sizeof(T));
    return SKIPPER_OK;
}
template <typename T>
static void free_arr(skipper_ctx *c, T *&p, size_t n) {
    dev_free(c, p, n * sizeof(T));
    p = nullptr;
}

// ------------------------------------------------------------------------------------ SST (Eq.5)
// numpy.percentile(a, p) with the default 'linear' method, replicated operation by operation:
// q = p / 100; vi = (n-1)*q; lo = floor(vi); g = vi - lo;
// lerp(a, b, g) = a + (b-a)*g, or b - (b-a)*(1-g) when g >= 0.5.
extern "C" double skipper_sst_host(const long long *s, int n, double p) {
    if (n <= 0) return NAN;
    std::vector<long long> v(s, s + n);
    std::sort(v.begin(), v.end());
    const double q = p / 100.0;
    const double vi = (double)(n - 1) * q;
    double lo_d = std::floor(vi);
    long long lo = (long long)lo_d;
    if (lo < 0) lo = 0;
    if (lo > n - 1) lo = n - 1;
    long long hi = std::min<long long>(lo + 1, n - 1);
    const double g = vi - lo_d;
    const long long diff = v[hi] - v[lo];
    const double a = (double)v[lo], b = (double)v[hi];
    if (g >= 0.5) return b - (double)diff * (1.0 - g);
    return a + (double)diff * g;
}

// the same on float64 values (the weighted SAM metric): lerp on doubles as numpy does
static double sst_double(const double *s, int n, double p) {
    if (n <= 0) return NAN;
    std::vector<double> v(s, s + n);
    std::sort(v.begin(), v.end());
    const double q = p / 100.0;
    const double vi = (double)(n - 1) * q;
    const double lo_d = std::floor(vi);
    long long lo = (long long)lo_d;
    if (lo < 0) lo = 0;
    if (lo > n - 1) lo = n - 1;
    const long long hi = std::min<long long>(lo + 1, n - 1);
    const double g = vi - lo_d;
    const double diff = v[hi] - v[lo];
    if (g >= 0.5) return v[hi] - diff * (1.0 - g);
    return v[lo] + diff * g;
}

// ------------------------------------------------------------------------------------ create
static skipper_status validate_and_shape(skipper_ctx *c, const skipper_layer *layers, int n) {
    if (!layers || n < 2) return fail(c, SKIPPER_EINVAL, "need at least one spiking layer and a readout");
    if (layers[n - 1].kind != SKIPPER_LAYER_READOUT) return fail(c, SKIPPER_EINVAL, "last layer must be the readout");
    c->L.resize(n);
    c->Ls = n - 1;
    for (int i = 0; i < n; ++i) {
        Layer &l = c->L[i];
        l.d = layers[i];
        const skipper_layer &d = layers[i];
        if (d.cin <= 0 || d.cout <= 0) return fail(c, SKIPPER_EINVAL, "layer %d: cin/cout must be positive", i);
        if (i < n - 1 && d.kind == SKIPPER_LAYER_READOUT) return fail(c, SKIPPER_EINVAL, "layer %d: readout must be last", i);
        if (d.kind == SKIPPER_LAYER_CONV3X3) {
            l.conv = true;
            l.H = d.h;
            l.W = d.w;
            l.Cin = d.cin;
            l.Cout = d.cout;
            l.stride = d.stride == 0 ? 1 : d.stride;
            if (l.stride != 1 && l.stride != 2) return fail(c, SKIPPER_EINVAL, "layer %d: stride must be 1 or 2", i);
            l.Hin = d.h * l.stride;
            l.Win = d.w * l.stride;
            l.pool = d.pool == 2;
            if (d.pool != 0 && d.pool != 2) return fail(c, SKIPPER_EINVAL, "layer %d: pool must be 0 or 2", i);
            if (l.pool && (d.h % 2 || d.w % 2)) return fail(c, SKIPPER_EINVAL, "layer %d: pooled size must be even", i);
            l.PH = l.pool ? d.h / 2 : d.h;
            l.PW = l.pool ? d.w / 2 : d.w;
            l.N = (long long)d.h * d.w * d.cout;
            l.Nout = (long long)l.PH * l.PW * d.cout;
            l.Nin = (long long)l.Hin * l.Win * d.cin;
            l.wcount = (size_t)d.cout * 9 * d.cin;
        } else if (d.kind == SKIPPER_LAYER_FC || d.kind == SKIPPER_LAYER_READOUT) {
            l.fc = d.kind == SKIPPER_LAYER_FC;
            l.readout = d.kind == SKIPPER_LAYER_READOUT;
            if (l.readout) {
                if (d.pool != 0 && d.pool != 1) return fail(c, SKIPPER_EINVAL, "readout: pool must be 0 or 1 (GAP)");
                l.gap = d.pool == 1;
            }
            l.Cin = d.cin;
            l.Cout = d.cout;
            l.N = l.Nout = d.cout;
            l.Nin = d.cin;
            l.wcount = (size_t)d.cout * d.cin;
        } else {
            return fail(c, SKIPPER_EINVAL, "layer %d: unknown kind %d", i, d.kind);
        }
        if (!l.readout) {
            if (!(d.theta > 0.f) || !(d.lambda > 0.f) || d.lambda > 1.f)
                return fail(c, SKIPPER_EINVAL, "layer %d: need theta > 0 and 0 < lambda <= 1 (Eq.1)", i);
            if (d.cout % 4) return fail(c, SKIPPER_EINVAL, "layer %d: cout must be a multiple of 4", i);
        }
    }
    // chaining
    const Layer &f = c->L[0];
    if (f.conv) {
        c->in_h = f.Hin;
        c->in_w = f.Win;
        c->in_c = f.Cin;
    } else {
        c->in_h = c->in_w = 1;
        c->in_c = f.Cin;
    }
    c->in_elems = (long long)c->in_h * c->in_w * c->in_c;
    c->in_row = c->in_elems;
    if (f.conv) {
        if (9 * f.Cin <= 64 && f.Cin % 64) {  // narrow input (RGB, DVS polarity): 3x3 im2col, K0 columns
            c->in_kind = 1;
            c->K0 = 9 * f.Cin <= 32 ? 32 : 64;
            c->in_row = (long long)f.H * f.W * c->K0;
        } else {
            c->in_kind = 2;
        }
    }
    for (int i = 1; i < n; ++i) {
        const Layer &p = c->L[i - 1];
        const Layer &l = c->L[i];
        if (l.conv) {
            if (!p.conv || l.Hin != p.PH || l.Win != p.PW || l.Cin != p.Cout)
                return fail(c, SKIPPER_EINVAL, "layer %d: conv input must be the %dx%dx%d output of layer %d", i, p.PH, p.PW,
                            p.Cout, i - 1);
        } else if (l.gap) {
            if (!p.conv || l.Cin != p.Cout)
                return fail(c, SKIPPER_EINVAL, "GAP readout: cin %d must be the channels of conv layer %d", l.Cin, i - 1);
        } else if (l.Cin != p.Nout) {
            return fail(c, SKIPPER_EINVAL, "layer %d: cin %d != %lld outputs of layer %d", i, l.Cin, p.Nout, i - 1);
        }
    }
    // residual shortcuts (reading 8): source r = i - 2, option A
    for (int i = 0; i < c->Ls; ++i) {
        Layer &l = c->L[i];
        const int r = layers[i].residual_from;
        if (r == -1) continue;
        if (!l.conv || r != i - 2 || r < 0)
            return fail(c, SKIPPER_EUNSUPPORTED, "layer %d: residual_from must be -1 or %d (a conv layer)", i, i - 2);
        Layer &src = c->L[r];
        if (!src.conv || src.pool || l.pool)
            return fail(c, SKIPPER_EUNSUPPORTED, "layer %d: residual between unpooled conv layers only", i);
        const int rs = src.H / l.H;
        if ((rs != 1 && rs != 2) || src.H != rs * l.H || src.W != rs * l.W || src.Cout > l.Cout ||
            (l.Cout - src.Cout) % 8)
            return fail(c, SKIPPER_EINVAL, "layer %d: option-A shortcut from %dx%dx%d to %dx%dx%d", i, src.H, src.W,
                        src.Cout, l.H, l.W, l.Cout);
        l.res = r;
        src.res_to = i;
    }
    // kernel support per layer
    for (int i = 0; i < c->Ls; ++i) {
        Layer &l = c->L[i];
        if (l.conv && i == 0 && c->in_kind == 1) {
            if (l.Cout % 8) return fail(c, SKIPPER_EUNSUPPORTED, "layer 0: cout %% 8 == 0");
            continue;
        }
        if (l.conv) {
            auto boxok = [](int h, int w, int rows) {
                if (w > rows || rows % w) return false;
                int by = rows / w;
                if (by <= h) return h % by == 0;
                return by % h == 0;
            };
            const bool implicit = l.Cin % 64 == 0 && (l.Cout % 64 == 0 || i == 0) && l.stride == 1 &&
                                  boxok(l.H, l.W, 128) && boxok(l.H, l.W, 64);
            if (!implicit) {  // explicit im2col + GEMM (narrow channels, stride 2, small images)
                if (i == 0) return fail(c, SKIPPER_EUNSUPPORTED, "layer 0: wide-input conv needs cin %% 64 == 0, stride 1");
                if (l.Cin % 8 || l.Cout % 8)
                    return fail(c, SKIPPER_EUNSUPPORTED, "layer %d: im2col conv needs cin, cout %% 8 == 0", i);
                l.icol = true;
                // the strided / narrow implicit conv (gemm_tc.cu plan_conv_s) where its boxes fit
                auto narrow_ok = [](int ch) { return ch == 16 || ch == 32 || ch % 64 == 0; };
                const bool tiles = boxok(l.H, l.W, 128) && l.W * l.stride <= 256 &&
                                   (128 / l.W <= l.H ? 128 / l.W : l.H) * l.stride <= 256;
                const char *en = getenv("SKIPPER_NO_NARROW_IMPLICIT");
                const bool allow = !(en && atoi(en));
                l.fwd_s = allow && tiles && narrow_ok(l.Cin);
                l.dgrad_s = allow && tiles && l.stride == 1 && narrow_ok(l.Cout);
                // the gather kernel where it measured faster than the TMA boxes (tools/conv_s_bench.py):
                // 16-channel inputs, and 32 -> <= 32
                auto gather_ok = [](int ci, int co, int st, int sg) {
                    return sk::conv_narrow_supported(ci, co, st, sg) && (ci == 16 || (ci == 32 && co <= 32));
                };
                l.fwd_g = allow && gather_ok(l.Cin, l.Cout, l.stride, 1);
                l.dgrad_g = allow && gather_ok(l.Cout, l.Cin, 1, -1) && l.stride == 1;
                if (l.fwd_g) l.fwd_s = false;
                const char *enl = getenv("SKIPPER_NO_NARROW_LIF");
                l.nlif = l.fwd_g && !l.pool && sk::conv_narrow_lif_supported(l.Cin, l.Cout, l.stride) && !(enl && atoi(enl));
                if (l.dgrad_g) l.dgrad_s = false;
            }
        } else {
            if (l.Cin % 8 || l.Cout % 8) return fail(c, SKIPPER_EUNSUPPORTED, "layer %d: fc needs cin, cout %% 8 == 0", i);
        }
    }
    if (c->L.back().readout && c->L.back().Cout > 1024) return fail(c, SKIPPER_EUNSUPPORTED, "readout classes <= 1024");
    return SKIPPER_OK;
}

static skipper_status zero_dev(skipper_ctx *c, void *p, size_t bytes) {
    if (p && bytes) CK(cudaMemsetAsync(p, 0, bytes, c->st));
    return SKIPPER_OK;
}

static long long max_nout(const skipper_ctx *c) {
    long long m = 0;
    for (int i = 0; i < c->Ls; ++i) m = std::max(m, c->L[i].Nout);
    return m;
}
static long long max_n(const skipper_ctx *c) {
    long long m = 0;
    for (int i = 0; i < c->Ls; ++i) m = std::max(m, c->L[i].N);
    return m;
}
static long long max_icol(const skipper_ctx *c) {  // im2col columns per sample-row (icol layers)
    long long m = 0;
    for (int i = 0; i < c->Ls; ++i)
        if (c->L[i].icol) m = std::max(m, (long long)c->L[i].H * c->L[i].W * 9 * c->L[i].Cin);
    return m;
}
// icol layers run in chunks of sample-rows so that the im2col / dgrad column buffers stay bounded
// (SKIPPER_ICOL_CHUNK_MB of bf16 columns, default 1024) however many rows a pass has.
static long long icol_chunk(const skipper_ctx *c) {
    static long long mb = -1;
    if (mb < 0) {
        const char *e = getenv("SKIPPER_ICOL_CHUNK_MB");
        mb = e ? std::max(1, atoi(e)) : 1024;
    }
    const long long per = max_icol(c) * 2;
    return per ? std::max(1LL, (mb << 20) / per) : 1;
}
static long long max_gemm_io(const skipper_ctx *c) {  // fp32 I (fwd) and g (dgrad) per sample-row
    long long m = 0;
    for (int i = 0; i < c->Ls; ++i) {
        m = std::max(m, c->L[i].N * c->L[i].fsplit);
        if (i > 0) m = std::max(m, c->L[i].Nin * c->L[i].dsplit);
    }
    return std::max(m, 4LL);
}

// Split-K for fc GEMMs whose output has too few 128 x BN tiles to fill the SMs (M = S*B rows is
// small).  Fixed per layer from the first-pass shape so the recompute reduces in the same order.
static int fc_splits(int M, int N, int K, int num_sms) {
    const int bn = N <= 64 ? 64 : (N <= 128 ? 128 : 256);
    const long long tiles = (long long)((M + 127) / 128) * ((N + bn - 1) / bn);
    const int kb = (K + 63) / 64;
    if (tiles >= num_sms || kb < 8) return 1;
    int s = (int)((num_sms + tiles - 1) / tiles);
    s = std::min(s, 8);
    s = std::min(s, kb / 4);
    return std::max(s, 1);
}

// First-pass arena layout for F segments per launch: only what the layers before the tail use - the output
// ring (the last of them writes into the tail's input rows), fp32 currents of the layers that run as GEMM +
// scan, the staged layer-0 operand when layer 0 is not the fused kernel, the im2col columns of icol layers -
// and the fc tail's chunk buffers (input rows, ping-pong outputs, currents with split partials).
struct FirstLayout {
    size_t pbytes = 0, ibytes = 0, xbytes = 0, cbytes = 0, tin = 0, tp = 0, ti = 0, total = 0;
};
static FirstLayout first_layout(const skipper_ctx *c, int F) {
    FirstLayout f;
    const size_t rowsB = (size_t)F * c->S * c->B;
    long long mo = 0, mio = 0, mic = 0;
    for (int i = 0; i < c->tail0; ++i) {
        const Layer &l = c->L[i];
        if (i < c->tail0 - 1 || c->tail0 == c->Ls) mo = std::max(mo, l.Nout);
        const bool kernel_lif = l.cfused || l.nlif || (i == 0 && c->l0_fused);
        if (!kernel_lif) mio = std::max(mio, l.N * l.fsplit);
        if (l.icol) mic = std::max(mic, (long long)l.H * l.W * 9 * l.Cin);
    }
    f.pbytes = al256(rowsB * mo * 2);
    f.ibytes = al256(rowsB * mio * 4);
    f.xbytes = (c->tail0 > 0 && !c->l0_fused) ? al256(rowsB * c->in_row * 2) : 0;
    if (c->tail0 < c->Ls) {
        const size_t rowsT = (size_t)c->tail_G * c->S * c->B;
        f.tin = al256(rowsT * (c->tail0 == 0 ? c->in_row : c->L[c->tail0 - 1].Nout) * 2);
        long long to = 0, ti = 0;
        for (int i = c->tail0; i < c->Ls; ++i) {
            to = std::max(to, c->L[i].Nout);
            ti = std::max(ti, c->L[i].N * c->L[i].fsplitT);
        }
        f.tp = al256(rowsT * to * 2);
        f.ti = al256(rowsT * ti * 4);
    }
    f.cbytes = al256(std::min<long long>(rowsB, icol_chunk(c)) * mic * 2);
    f.total = c->nP * f.pbytes + f.ibytes + f.xbytes + f.cbytes + f.tin + 2 * f.tp + f.ti;
    return f;
}

// RECOMPUTE / RECORD arena for R rows: per-layer stored U and outputs, fp32 I/g, bf16 delta ring, staged
// layer-0 operand, icol columns
static size_t rows_bytes(const skipper_ctx *c, int R) {
    const size_t rowsB = (size_t)R * c->B;
    size_t bytes = 0;
    for (int i = 0; i < c->Ls; ++i) bytes += al256(rowsB * c->L[i].Nout * 2) + al256(rowsB * c->L[i].N * 4);
    const long long ch = std::min<long long>(rowsB, icol_chunk(c));
    bytes += al256(rowsB * max_gemm_io(c) * 4) + c->nD * (al256(rowsB * max_n(c) * 2) + al256(ch * max_icol(c) * 2)) +
             al256(rowsB * c->in_row * 2) + al256(ch * max_icol(c) * 4);
    return bytes;
}

extern "C" skipper_status skipper_create(const skipper_layer *layers, int n_layers, const skipper_config *cfg,
                                         const skipper_allocator *alloc, void *cuda_stream, skipper_ctx **out) {
    if (out) *out = nullptr;
    if (!cfg || !out) return fail(nullptr, SKIPPER_EINVAL, "null config or output pointer");
    skipper_ctx *c = new skipper_ctx();
    auto bail = [&](skipper_status s) {
        g_last_error = c->err.empty() ? g_last_error : c->err;
        skipper_destroy(c);
        return s;
    };
    c->cfg = *cfg;
    c->st = static_cast<cudaStream_t>(cuda_stream);
    if (alloc && alloc->alloc && alloc->free) {
        c->alloc = *alloc;
        c->own_alloc = false;
    }
    skipper_status s = validate_and_shape(c, layers, n_layers);
    if (s != SKIPPER_OK) return bail(s);
    c->T = cfg->T;
    c->B = cfg->batch;
    c->Bg = cfg->global_batch > 0 ? cfg->global_batch : cfg->batch;
    if (c->T <= 0 || c->B <= 0) return bail(fail(c, SKIPPER_EINVAL, "T and batch must be positive"));
    if (cfg->mode < 0 || cfg->mode > 3) return bail(fail(c, SKIPPER_EINVAL, "unknown mode %d", cfg->mode));
    if (cfg->surrogate != SKIPPER_SURR_TRIANGLE && cfg->surrogate != SKIPPER_SURR_FAST_SIGMOID)
        return bail(fail(c, SKIPPER_EINVAL, "unknown surrogate %d", cfg->surrogate));
    if (cfg->sam != SKIPPER_SAM_SPIKES && cfg->sam != SKIPPER_SAM_WEIGHTED && cfg->sam != SKIPPER_SAM_L2TRACE)
        return bail(fail(c, SKIPPER_EINVAL, "unknown SAM metric %d", cfg->sam));
    if (cfg->mode == SKIPPER_MODE_FULL) {
        c->C = 1;
    } else if (cfg->mode == SKIPPER_MODE_TBPTT) {
        c->C = cfg->C;
        if (c->C <= 0 || c->T % c->C)
            return bail(fail(c, SKIPPER_EINVAL, "C=%d truncation windows must divide T=%d", c->C, c->T));
    } else {
        c->C = cfg->C;
        if (c->C <= 0 || c->T % c->C)
            return bail(fail(c, SKIPPER_EINVAL, "C=%d must divide T=%d (P:1779-1781)", c->C, c->T));
        const int Ln = n_layers;
        if (c->T / c->C <= Ln)
            return bail(fail(c, SKIPPER_EINVAL, "segment length T/C=%d must exceed the %d layers (P:840-853)", c->T / c->C, Ln));
        if (!(cfg->p >= 0.0 && cfg->p < 100.0))
            return bail(fail(c, SKIPPER_EINVAL, "p=%g outside [0, 100) (Eq.5)", cfg->p));
        if (cfg->mode == SKIPPER_MODE_SKIP && cfg->p / 100.0 > 1.0 - (double)c->C * Ln / c->T) {
            char buf[256];
            snprintf(buf, sizeof buf, "warning: p=%g exceeds the Eq.7 rule of thumb p_max=%g (P:1082-1091)", cfg->p,
                     100.0 * (1.0 - (double)c->C * Ln / c->T));
            c->err = buf;
        }
    }
    c->S = c->T / c->C;
    c->G = (cfg->mode == SKIPPER_MODE_CKPT || cfg->mode == SKIPPER_MODE_SKIP) ? std::max(1, std::min(cfg->group, c->C)) : 1;
    {
        // opt-in (SKIPPER_WGRAD_OVERLAP=1): measured +0.4 % on cfg 2 and -2 % on cfg 3 for one
        // more copy of the layer outputs - the GPU is saturated, the weight gradients cost SM time wherever they run
        const char *e = getenv("SKIPPER_WGRAD_OVERLAP");
        c->wdb = (cfg->mode == SKIPPER_MODE_CKPT || cfg->mode == SKIPPER_MODE_SKIP) && c->G == 1 && c->C > 1 &&
                 (e && atoi(e));
    }
    c->num_sms = sk::device_num_sms();
    c->host_prof = getenv("SKIPPER_HOST_PROFILE") && atoi(getenv("SKIPPER_HOST_PROFILE"));
    if (cudaStreamCreateWithFlags(&c->st2, cudaStreamNonBlocking) != cudaSuccess)
        return bail(fail(c, SKIPPER_ECUDA, "side stream creation failed"));
    for (int i = 0; i < c->Ls; ++i)
        if (c->L[i].res >= 0) c->nD = c->nP = 3;
    for (int k = 0; k < 3; ++k)
        if (cudaEventCreateWithFlags(&c->ev_ready[k], cudaEventDisableTiming) != cudaSuccess ||
            cudaEventCreateWithFlags(&c->ev_done[k], cudaEventDisableTiming) != cudaSuccess)
            return bail(fail(c, SKIPPER_ECUDA, "event creation failed"));
    for (int k = 0; k < 2; ++k)
        if (cudaEventCreateWithFlags(&c->ev_slot[k], cudaEventDisableTiming) != cudaSuccess)
            return bail(fail(c, SKIPPER_ECUDA, "event creation failed"));
    {
        const Layer &f = c->L[0];
        const char *e = getenv("SKIPPER_NO_L0_FUSION");
        c->l0_fused = c->in_kind == 1 && c->K0 == 32 && c->Ls >= 2 && !(e && atoi(e)) && f.stride == 1 &&
                      sk::layer0_supported(c->B, f.H, f.W, f.Cin, f.Cout, f.pool ? 1 : 0);
        // opt-in: measured slower than reverse scan + im2col wgrad GEMM on VGG-5
        const char *e2 = getenv("SKIPPER_L0_BWD_FUSION");
        c->l0_bwd_fused = c->l0_fused && (e2 && atoi(e2)) && cfg->mode != SKIPPER_MODE_TBPTT &&
                          sk::layer0_bwd_supported(c->B, f.H, f.W, f.Cin, f.Cout, f.pool ? 1 : 0);
        // conv layers after the first: tensor-core GEMM + LIF scan fused (not the last spiking layer,
        // whose scan also accumulates the readout counts)
        // The fused kernel's work unit is (128 pixels of one timestep, <= 128 channels) walking the rows of
        // the segment in order, so its parallelism is the unit count alone: deep layers at small spatial
        // size (VGG-11 at 4x4 / 2x2: 16-64 units) would leave most SMs idle for a long sequential K loop.
        // Those run layer-major instead (one GEMM over all rows of the segment, then the scan).
        const char *e3 = getenv("SKIPPER_NO_CONV_FUSION");
        const char *e4 = getenv("SKIPPER_CL_MIN_UNITS");
        const int min_units = e4 ? atoi(e4) : (c->num_sms * 4) / 5;
        for (int i = 1; i < c->Ls - 1; ++i) {
            Layer &l = c->L[i];
            const long long units = ((long long)c->B * l.H * l.W + 127) / 128 * (l.Cout == 64 ? 1 : l.Cout / 128);
            l.cfused = l.conv && !l.icol && l.res < 0 && !(e3 && atoi(e3)) && units >= min_units &&
                       sk::conv_lif_supported(c->B, l.H, l.W, l.Cin, l.Cout, l.pool ? 1 : 0);
        }
        // dgrad of layer i with layer i-1's reverse scan fused (conv_lif.cu BWD): stride-1 3x3 layer i whose
        // input is layer i-1's unpooled output, layer i-1 neither a shortcut source nor layer 0's fused
        // backward; units = (128-pixel tile, 64 channels of C_{i-1}) as the forward's fill rule
        // opt-in (SKIPPER_BWD_FUSION=1): the fused kernel is faster than the dgrad GEMM + reverse scan it replaces
        // (cfg 2: 0.45 vs 0.72 ms per step serialised) but the step is not (the backward's
        // critical path is shared with the side-stream weight gradients)
        const char *e5 = getenv("SKIPPER_BWD_FUSION");
        for (int i = 1; i < c->Ls; ++i) {
            Layer &l = c->L[i];
            const Layer &pv = c->L[i - 1];
            const long long units = ((long long)c->B * l.H * l.W + 127) / 128 * (pv.Cout % 128 ? pv.Cout / 64 : pv.Cout / 128);
            l.dlif = (e5 && atoi(e5)) && l.conv && !l.icol && l.stride == 1 && pv.conv && !pv.icol && !pv.pool &&
                     pv.res_to < 0 && !(i == 1 && c->l0_bwd_fused) && pv.H == l.H && pv.W == l.W &&
                     units >= min_units && sk::conv_lif_bwd_supported(c->B, l.H, l.W, l.Cout, l.Cin);
        }
    }
    for (int i = 0; i < c->Ls; ++i) {
        Layer &l = c->L[i];
        if (!l.fc) continue;
        const int rowsM = c->S * c->B;
        l.fsplit = fc_splits(rowsM, l.Cout, l.Cin, c->num_sms);
        if (i > 0) l.dsplit = fc_splits(rowsM, l.Cin, l.Cout, c->num_sms);
    }
    // The fc tail (a few thousand neurons per sample) would run as tiny latency-bound launches per
    // segment; in the first pass it is evaluated layer-major over chunks of tail_G segments instead (its
    // recurrences still run in time order; checkpoints are written every S rows).  The T*B rows are cut into
    // ceil(T*B / SKIPPER_TAIL_ROWS) balanced chunks of whole segments (default 8192 sample-rows: the whole
    // sequence at cfg 2): at most max(8192, S*B) rows, so the tail's buffers do not grow with T (a whole-sequence tail held an
    // O(T * B) activation term that checkpointing never released).
    c->tail0 = c->Ls;
    while (c->tail0 > 0 && c->L[c->tail0 - 1].fc) --c->tail0;
    if (cfg->mode == SKIPPER_MODE_FULL || cfg->mode == SKIPPER_MODE_TBPTT) c->tail0 = c->Ls;
    {
        const char *e = getenv("SKIPPER_TAIL_ROWS");
        const long long target = e ? std::max(1, atoi(e)) : 8192;
        const long long rows = (long long)c->T * c->B;
        const long long nchunks = std::max<long long>(1, (rows + target - 1) / target);
        c->tail_G = (int)std::max<long long>(1, (c->C + nchunks - 1) / nchunks);  // balanced chunks
        for (int i = c->tail0; i < c->Ls; ++i)
            c->L[i].fsplitT = fc_splits(c->tail_G * c->S * c->B, c->L[i].Cout, c->L[i].Cin, c->num_sms);
        // The first pass of the layers before the tail runs F segments per launch (checkpoints every S rows
        // inside the kernels): fewer launches, each amortising its fixed cost (prologue, pipeline fill, state
        // load / store) over more rows.  F * S * B <= SKIPPER_FIRST_ROWS (default 4096) sample-rows of
        // first-pass buffers - a constant, so Eq.3's O(C) + O(S) law is kept.
        // Bounded also so that the first-pass arena stays below the recompute arena of the expected kept rows
        // ((1 - p/100)(S - 1) + 1): the step's peak memory stays the paper's (Eq.3 / Eq.6), F only spends
        // memory the backward would claim anyway.
        const char *ef = getenv("SKIPPER_FIRST_ROWS");
        const long long frows = ef ? std::max(1, atoi(ef)) : 4096;
        if (cfg->mode == SKIPPER_MODE_CKPT || cfg->mode == SKIPPER_MODE_SKIP) {
            const int kexp = cfg->mode == SKIPPER_MODE_SKIP
                                 ? std::min(c->S, 1 + (int)std::ceil((1.0 - cfg->p / 100.0) * (c->S - 1)))
                                 : c->S;
            const size_t cap = rows_bytes(c, kexp);
            c->F = 1;
            while (c->F < c->C && (long long)(c->F + 1) * c->S * c->B <= frows &&
                   first_layout(c, c->F + 1).total <= cap)
                ++c->F;
        }
    }

    // ---- persistent allocations
    c->dw_total = 0;
    for (auto &l : c->L) c->dw_total += l.wcount;
#define AL(ptr, n)                                  \
    do {                                            \
        s = alloc_arr(c, &(ptr), (size_t)(n));      \
        if (s != SKIPPER_OK) return bail(s);        \
    } while (0)
    AL(c->dw_all, c->dw_total);
    size_t off = 0;
    for (int i = 0; i < (int)c->L.size(); ++i) {
        Layer &l = c->L[i];
        AL(l.w, l.wcount);
        AL(l.m, l.wcount);
        AL(l.v, l.wcount);
        AL(l.wb, l.wcount);
        l.dw = c->dw_all + off;
        off += l.wcount;
        if (!l.readout) {
            if (i > 0) AL(l.wt, l.wcount);
            if (i == 0 && c->in_kind == 1) {
                AL(l.wbp, (size_t)l.Cout * c->K0);
                AL(l.dwp, (size_t)l.Cout * c->K0);
            }
            const size_t bn = (size_t)c->B * l.N;
            l.sbn = l.cfused ? (size_t)sk::conv_lif_state_count(c->B, l.H, l.W, l.Cout)
                    : (i == 0 && c->l0_fused) ? (size_t)sk::layer0_state_count(c->B, l.H, l.W, l.Cout, l.pool ? 1 : 0)
                                              : bn;
            AL(l.U_run, l.sbn);
            AL(l.o_run, l.sbn);
            AL(l.carry, bn);
            if (cfg->mode != SKIPPER_MODE_FULL && cfg->mode != SKIPPER_MODE_TBPTT) {
                AL(l.ckU, l.sbn * c->C);
                AL(l.cko, l.sbn * c->C);
            }
            if (cfg->debug_record) {
                for (int k = 0; k < 2; ++k) {
                    AL(l.dbg[k], bn * c->T);
                    AL(l.dbgo[k], bn * c->T);
                }
            }
        }
    }
    AL(c->s_part, (size_t)(c->Ls + 1) * c->T * 32);  // [layer group][T][32] partial counters
    if (cfg->sam == SKIPPER_SAM_L2TRACE) {
        AL(c->u2_part, (size_t)c->T * 32);
        AL(c->u2_dev, (size_t)c->T);
    }
    AL(c->s_dev, (size_t)(c->Ls + 1) * c->T);
    const Layer &last = c->L[c->Ls - 1];
    const Layer &ro = c->L.back();
    AL(c->cnt, (size_t)c->B * last.Nout);
    if (ro.gap) {
        AL(c->cnt_gap, (size_t)c->B * ro.Cin);
        AL(c->g_gap, (size_t)c->B * ro.Cin);
    }
    AL(c->cnt_kept, (size_t)c->B * last.Nout);
    AL(c->g_last, (size_t)c->B * last.Nout);
    AL(c->z, (size_t)c->B * ro.Cout);
    AL(c->dz, (size_t)c->B * ro.Cout);
    AL(c->loss_dev, 1);
    AL(c->kept_dev, (size_t)c->T);
    AL(c->grp_dev, (size_t)c->T);
    // split-K slices of the weight gradients: the split count of every wgrad launch is at most the count the
    // plan chooses at the layer's largest reduction (T rows in FULL mode, G*S otherwise), which sizes the slices
    {
        const long long Rmax = cfg->mode == SKIPPER_MODE_FULL ? c->T : (long long)c->S * c->G;  // rows per backward
        const long long nbmax = Rmax * c->B;
        const bool nw_off = getenv("SKIPPER_NO_NARROW_WGRAD") && atoi(getenv("SKIPPER_NO_NARROW_WGRAD"));
        // experiments: SKIPPER_WGRAD_ATOMIC=1 = the round-1 nondeterministic reduce-add into dW
        const bool atomic_wg = getenv("SKIPPER_WGRAD_ATOMIC") && atoi(getenv("SKIPPER_WGRAD_ATOMIC"));
        for (int i = 0; i < c->Ls; ++i) {
            Layer &l = c->L[i];
            l.wg_count = l.wcount;
            int ns = 0;
            if (i == 0 && c->l0_bwd_fused) {
                ns = 0;
            } else if (l.icol && !nw_off && sk::narrow_wgrad_supported(l.Cin, l.Cout, l.stride, l.H, l.W)) {
                ns = sk::narrow_wgrad_slices(l.Cin, l.Cout, l.stride, l.H, l.W, c->num_sms);
                l.wsl_narrow = true;
                if (ns < 1) return bail(fail(c, SKIPPER_ECUDA, "narrow weight-gradient occupancy query failed"));
            } else if (l.icol) {
                ns = sk::fc_wgrad_splits(std::min<long long>(nbmax, icol_chunk(c)) * l.H * l.W, l.Cout, 9 * l.Cin,
                                         c->num_sms);
            } else if (i == 0 && c->in_kind == 1) {
                ns = sk::fc_wgrad_splits(nbmax * l.H * l.W, l.Cout, c->K0, c->num_sms);
                l.wg_count = (size_t)l.Cout * c->K0;
            } else if (l.conv) {
                ns = sk::conv_wgrad_splits(nbmax * l.H * l.W, l.Cin, l.Cout, c->num_sms);
            } else {
                ns = sk::fc_wgrad_splits(nbmax, l.Cout, l.Cin, c->num_sms);
            }
            if (atomic_wg && !l.wsl_narrow) ns = 0;   // legacy: split-K reduce-add straight into dW
            l.wsl = ns;                               // 1: unsplit, reduce-add into dW (one writer per launch)
            if (ns > 1 || l.wsl_narrow) {
                l.wsl = ns;
                AL(l.dws, (size_t)ns * l.wg_count);
                s = zero_dev(c, l.dws, (size_t)ns * l.wg_count * 4);
                if (s != SKIPPER_OK) return bail(s);
            }
        }
    }
#undef AL
    for (auto &l : c->L) {
        s = zero_dev(c, l.w, l.wcount * 4);
        if (s == SKIPPER_OK) s = zero_dev(c, l.m, l.wcount * 4);
        if (s == SKIPPER_OK) s = zero_dev(c, l.v, l.wcount * 4);
        if (s == SKIPPER_OK) s = zero_dev(c, l.wb, l.wcount * 2);
        if (s == SKIPPER_OK && l.wt) s = zero_dev(c, l.wt, l.wcount * 2);
        if (s != SKIPPER_OK) return bail(s);
    }
    s = zero_dev(c, c->dw_all, c->dw_total * 4);
    if (s != SKIPPER_OK) return bail(s);
    if (cudaStreamSynchronize(c->st) != cudaSuccess) return bail(fail(c, SKIPPER_ECUDA, "stream sync failed at create"));
    c->s_host.assign(c->T, 0);
    c->counts_host.assign((size_t)(c->Ls + 1) * c->T, 0);
    c->sam_host.assign(c->T, 0.0);
    c->keep.assign(c->T, 1);
    c->sst.assign(c->C, NAN);
    *out = c;
    return SKIPPER_OK;
}

extern "C" void skipper_destroy(skipper_ctx *c) {
    if (!c) return;
    if (c->hp_ev[0]) cudaEventDestroy(c->hp_ev[0]);
    if (c->hp_ev[1]) cudaEventDestroy(c->hp_ev[1]);
    if (c->host_prof && c->hp_steps)
        fprintf(stderr, "skipper host profile: %lld steps, per step: first-pass issue %.3f ms, mask sync wait %.3f ms, "
                        "recompute+backward issue %.3f ms, device idle at the mask sync %.4f ms\n", c->hp_steps,
                c->hp_first / c->hp_steps, c->hp_sync / c->hp_steps, c->hp_bwd / c->hp_steps, c->hp_gap / c->hp_steps);
    if (c->st) cudaStreamSynchronize(c->st);
    if (c->arena) dev_free(c, c->arena, c->arena_bytes);
    for (auto &l : c->L) {
        dev_free(c, l.w, l.wcount * 4);
        dev_free(c, l.m, l.wcount * 4);
        dev_free(c, l.v, l.wcount * 4);
        dev_free(c, l.wb, l.wcount * 2);
        dev_free(c, l.wt, l.wcount * 2);
        dev_free(c, l.wbp, (size_t)l.Cout * c->K0 * 2);
        dev_free(c, l.dwp, (size_t)l.Cout * c->K0 * 4);
        if (!l.readout) {
            const size_t bn = (size_t)c->B * l.N;
            dev_free(c, l.U_run, l.sbn * 4);
            dev_free(c, l.o_run, l.sbn);
            dev_free(c, l.carry, bn * 4);
            dev_free(c, l.dws, (size_t)l.wsl * l.wg_count * 4);
            dev_free(c, l.ckU, l.sbn * c->C * 4);
            dev_free(c, l.cko, l.sbn * c->C);
            for (int k = 0; k < 2; ++k) {
                dev_free(c, l.dbg[k], bn * c->T * 4);
                dev_free(c, l.dbgo[k], bn * c->T);
            }
        }
    }
    dev_free(c, c->dw_all, c->dw_total * 4);
    if (!c->L.empty() && c->Ls > 0) {
        const Layer &last = c->L[c->Ls - 1];
        const Layer &ro = c->L.back();
        dev_free(c, c->s_part, (size_t)(c->Ls + 1) * c->T * 32 * 4);
        dev_free(c, c->u2_part, (size_t)c->T * 32 * 8);
        dev_free(c, c->u2_dev, (size_t)c->T * 8);
        dev_free(c, c->s_dev, (size_t)(c->Ls + 1) * c->T * 8);
        dev_free(c, c->cnt, (size_t)c->B * last.Nout * 4);
        dev_free(c, c->cnt_gap, (size_t)c->B * ro.Cin * 4);
        dev_free(c, c->g_gap, (size_t)c->B * ro.Cin * 4);
        dev_free(c, c->cnt_kept, (size_t)c->B * last.Nout * 4);
        dev_free(c, c->g_last, (size_t)c->B * last.Nout * 4);
        dev_free(c, c->z, (size_t)c->B * ro.Cout * 4);
        dev_free(c, c->dz, (size_t)c->B * ro.Cout * 4);
        dev_free(c, c->loss_dev, 4);
        dev_free(c, c->kept_dev, (size_t)c->T * 4);
        dev_free(c, c->grp_dev, (size_t)c->T * 4);
        dev_free(c, c->x_stage, (size_t)c->T * c->B * c->in_elems);
        dev_free(c, c->y_stage, (size_t)c->B * 4);
        dev_free(c, c->x_enc, (size_t)c->T * c->B * c->in_elems);
        dev_free(c, c->img_stage, (size_t)c->B * c->in_elems * 4);
        dev_free(c, c->rates_stage, (size_t)c->T * 4);
    }
    if (c->st) cudaStreamSynchronize(c->st);
    for (auto e : c->ev_pool) cudaEventDestroy(e);
    if (c->st2) {
        cudaStreamSynchronize(c->st2);
        cudaStreamDestroy(c->st2);
    }
    for (int k = 0; k < 3; ++k) {
        if (c->ev_ready[k]) cudaEventDestroy(c->ev_ready[k]);
        if (c->ev_done[k]) cudaEventDestroy(c->ev_done[k]);
    }
    for (int k = 0; k < 2; ++k)
        if (c->ev_slot[k]) cudaEventDestroy(c->ev_slot[k]);
    if (c->st3) {
        cudaStreamSynchronize(c->st3);
        cudaStreamDestroy(c->st3);
    }
    if (c->ev_w) cudaEventDestroy(c->ev_w);
    if (c->ev_comm) cudaEventDestroy(c->ev_comm);
    c->comm.destroy();
    delete c;
}

extern "C" const char *skipper_last_error(const skipper_ctx *c) {
    if (c) return c->err.c_str();
    return g_last_error.c_str();
}

extern "C" const char *skipper_status_string(int s) {
    switch (s) {
        case SKIPPER_OK: return "ok";
        case SKIPPER_EINVAL: return "invalid argument";
        case SKIPPER_ENOMEM: return "out of device memory";
        case SKIPPER_ECUDA: return "CUDA error";
        case SKIPPER_ENCCL: return "NCCL error";
        case SKIPPER_EORDER: return "call order violation";
        case SKIPPER_EFAILED: return "context failed earlier";
        case SKIPPER_EUNSUPPORTED: return "unsupported geometry";
    }
    return "unknown";
}

extern "C" const char *skipper_build_info(void) {
    return "skipper-b200: sm_100a tcgen05/TMA GEMMs, fused LIF scans; built " __DATE__ " " __TIME__;
}

// ------------------------------------------------------------------------------------ weights
static skipper_status check_ctx(skipper_ctx *c) {
    if (!c) return fail(nullptr, SKIPPER_EINVAL, "null context");
    if (c->poisoned) return SKIPPER_EFAILED;
    return SKIPPER_OK;
}

static skipper_status refresh_shadows(skipper_ctx *c, int i) {
    Layer &l = c->L[i];
    CK(sk::launch_cast_bf16(l.w, l.wb, l.wcount, c->st));
    if (l.wbp) CK(sk::launch_cast_pad_bf16(l.w, l.wbp, l.Cout, (int)(l.wcount / l.Cout), c->K0, c->st));
    if (l.wt) {
        if (l.conv)  // wt[ci][tap][co] = wb[co][tap][ci]
            CK(sk::launch_transpose_bf16(l.wb, l.wt, l.Cout, 9, l.Cin, c->st));
        else  // wt[k][n] = wb[n][k]
            CK(sk::launch_transpose_bf16(l.wb, l.wt, l.Cout, 1, l.Cin, c->st));
    }
    return SKIPPER_OK;
}

extern "C" size_t skipper_weight_count(const skipper_ctx *c, int layer) {
    if (!c || layer < 0 || layer >= (int)c->L.size()) return 0;
    return c->L[layer].wcount;
}

extern "C" skipper_status skipper_set_weights(skipper_ctx *c, int layer, const float *w_dev) {
    CKS(check_ctx(c));
    if (layer < 0 || layer >= (int)c->L.size() || !w_dev) return fail(c, SKIPPER_EINVAL, "bad layer or pointer");
    Layer &l = c->L[layer];
    CK(cudaMemcpyAsync(l.w, w_dev, l.wcount * 4, cudaMemcpyDeviceToDevice, c->st));
    return refresh_shadows(c, layer);
}

extern "C" skipper_status skipper_get_weights(skipper_ctx *c, int layer, float *w_dev) {
    CKS(check_ctx(c));
    if (layer < 0 || layer >= (int)c->L.size() || !w_dev) return fail(c, SKIPPER_EINVAL, "bad layer or pointer");
    CK(cudaMemcpyAsync(w_dev, c->L[layer].w, c->L[layer].wcount * 4, cudaMemcpyDeviceToDevice, c->st));
    return SKIPPER_OK;
}

extern "C" skipper_status skipper_get_grads(skipper_ctx *c, int layer, float *dw_dev) {
    CKS(check_ctx(c));
    if (layer < 0 || layer >= (int)c->L.size() || !dw_dev) return fail(c, SKIPPER_EINVAL, "bad layer or pointer");
    CK(cudaMemcpyAsync(dw_dev, c->L[layer].dw, c->L[layer].wcount * 4, cudaMemcpyDeviceToDevice, c->st));
    return SKIPPER_OK;
}

// ------------------------------------------------------------------------------------ arenas
// FIRST pass: two ping-pong output buffers of S rows and the fp32 current buffer.
// RECOMPUTE/RECORD (R rows): per-layer U and output rows, fp32 I/g, bf16 delta, gathered input.
static skipper_status arena_free(skipper_ctx *c) {
    if (c->arena) dev_free(c, c->arena, c->arena_bytes);
    c->arena = nullptr;
    c->arena_bytes = 0;
    for (auto &l : c->L) {
        l.Po = l.PoS[0] = l.PoS[1] = nullptr;
        l.Useg = nullptr;
    }
    c->xgS[0] = c->xgS[1] = nullptr;
    c->slot_rec[0] = c->slot_rec[1] = false;
    c->cur_slot = 0;
    c->I_buf = nullptr;
    c->d_buf = nullptr;
    for (int k = 0; k < 3; ++k) c->d_buf2[k] = c->P2[k] = c->cols[k] = nullptr;
    c->dcols = nullptr;
    c->xg = nullptr;
    c->tail_in = c->tailP[0] = c->tailP[1] = nullptr;
    c->tail_I = nullptr;
    return SKIPPER_OK;
}

// [s0, end) of the first-pass chunk starting at segment s0: F segments, never across an fc-tail chunk border
static int first_chunk_end(const skipper_ctx *c, int s0) {
    int end = std::min(c->C, s0 + c->F);
    if (c->tail0 < c->Ls) end = std::min(end, (s0 / c->tail_G + 1) * c->tail_G);
    return end;
}

static skipper_status arena_first(skipper_ctx *c) {
    arena_free(c);
    const FirstLayout f = first_layout(c, c->F);
    const int nP = c->nP;
    c->arena_bytes = f.total;
    c->arena = dev_alloc(c, c->arena_bytes);
    if (!c->arena) return fail(c, SKIPPER_ENOMEM, "first-pass arena of %zu bytes", c->arena_bytes);
    char *p = static_cast<char *>(c->arena);
    for (int k = 0; k < nP; ++k) c->P2[k] = reinterpret_cast<uint16_t *>(p + k * f.pbytes);
    c->I_buf = reinterpret_cast<float *>(p + nP * f.pbytes);
    c->xg = reinterpret_cast<uint16_t *>(p + nP * f.pbytes + f.ibytes);
    c->cols[0] = f.cbytes ? reinterpret_cast<uint16_t *>(p + nP * f.pbytes + f.ibytes + f.xbytes) : nullptr;
    char *q = p + nP * f.pbytes + f.ibytes + f.xbytes + f.cbytes;
    c->tail_in = f.tin ? reinterpret_cast<uint16_t *>(q) : nullptr;
    c->tailP[0] = f.tp ? reinterpret_cast<uint16_t *>(q + f.tin) : nullptr;
    c->tailP[1] = f.tp ? reinterpret_cast<uint16_t *>(q + f.tin + f.tp) : nullptr;
    c->tail_I = f.ti ? reinterpret_cast<float *>(q + f.tin + 2 * f.tp) : nullptr;
    return SKIPPER_OK;
}

static skipper_status arena_rows(skipper_ctx *c, int R) {
    arena_free(c);
    const size_t rowsB = (size_t)R * c->B;
    size_t bytes = 0;
    const int nslot = c->wdb ? 2 : 1;
    for (int i = 0; i < c->Ls; ++i) bytes += nslot * al256(rowsB * c->L[i].Nout * 2) + al256(rowsB * c->L[i].N * 4);
    const size_t ibytes = al256(rowsB * max_gemm_io(c) * 4);
    const size_t dbytes = al256(rowsB * max_n(c) * 2);
    const size_t xbytes = al256(rowsB * c->in_row * 2);
    const long long ch = std::min<long long>(rowsB, icol_chunk(c));
    const size_t cbytes = al256(ch * max_icol(c) * 2), dcbytes = al256(ch * max_icol(c) * 4);
    bytes += ibytes + c->nD * (dbytes + cbytes) + nslot * xbytes + dcbytes;
    c->arena_bytes = bytes;
    c->arena = dev_alloc(c, bytes);
    if (!c->arena) return fail(c, SKIPPER_ENOMEM, "segment arena of %zu bytes (%d rows)", bytes, R);
    char *p = static_cast<char *>(c->arena);
    for (int i = 0; i < c->Ls; ++i) {
        Layer &l = c->L[i];
        for (int k = 0; k < nslot; ++k) {
            l.PoS[k] = reinterpret_cast<uint16_t *>(p);
            p += al256(rowsB * l.Nout * 2);
        }
        l.Po = l.PoS[0];
        l.Useg = reinterpret_cast<float *>(p);
        p += al256(rowsB * l.N * 4);
    }
    c->I_buf = reinterpret_cast<float *>(p);
    p += ibytes;
    c->d_buf = reinterpret_cast<uint16_t *>(p);
    for (int k = 0; k < c->nD; ++k) c->d_buf2[k] = reinterpret_cast<uint16_t *>(p + k * dbytes);
    p += c->nD * dbytes;
    for (int k = 0; k < nslot; ++k) {
        c->xgS[k] = reinterpret_cast<uint16_t *>(p);
        p += xbytes;
    }
    c->xg = c->xgS[0];
    for (int k = 0; k < c->nD; ++k) c->cols[k] = cbytes ? reinterpret_cast<uint16_t *>(p + k * cbytes) : nullptr;
    p += c->nD * cbytes;
    c->dcols = dcbytes ? reinterpret_cast<float *>(p) : nullptr;
    return SKIPPER_OK;
}

// ------------------------------------------------------------------------------------ GEMM dispatch
// Cached GEMM plan: builds (and encodes the tensor maps) on first use of a (pointers, shape) key.
static bool get_plan(skipper_ctx *c, const PlanKey &k, sk::GemmLaunch &g, const std::function<bool(sk::GemmLaunch *)> &make) {
    auto it = c->plans.find(k);
    if (it != c->plans.end()) {
        g = it->second;
        return true;
    }
    if (!make(&g)) return false;
    if (c->plans.size() > 4096) c->plans.clear();
    c->plans.emplace(k, g);
    return true;
}

static skipper_status run_gemm(skipper_ctx *c, const sk::GemmLaunch &g, bool ok, const char *what, int layer,
                               int cls, double bytes, double flops, cudaStream_t s = nullptr) {
    if (!ok) return fail(c, SKIPPER_EUNSUPPORTED, "layer %d: cannot plan %s GEMM (tensor map)", layer, what);
    if (!s) s = c->st;
    // timing experiment only (gradients are wrong when set): SKIPPER_DIAG_NO_WGRAD=1 skips the weight-gradient
    // GEMMs, to measure how much of the step they hold on the critical path
    static const bool no_wgrad = getenv("SKIPPER_DIAG_NO_WGRAD") && atoi(getenv("SKIPPER_DIAG_NO_WGRAD"));
    if (no_wgrad && cls == K_GEMM_WGRAD) return SKIPPER_OK;
    ProfScope ps(c, cls, bytes, flops, s);
    CK(sk::gemm_run(g, s, c->num_sms));
    return SKIPPER_OK;
}

// conv_narrow.cu arguments for layer l: forward (X = the layer input, Wk = wb) or stride-1 dgrad (X = delta,
// Wk = the transposed shadow wt, output channels = the layer's cin)
static sk::NarrowConvArgs narrow_args(const Layer &l, const uint16_t *X, const uint16_t *Wk, float *Y, int nb, int sign) {
    sk::NarrowConvArgs a{};
    a.X = X;
    a.Wk = Wk;
    a.Y = Y;
    a.nb = nb;
    a.H = l.H;
    a.W = l.W;
    a.Hin = sign > 0 ? l.Hin : l.H;
    a.Win = sign > 0 ? l.Win : l.W;
    a.Cin = sign > 0 ? l.Cin : l.Cout;
    a.Cout = sign > 0 ? l.Cout : l.Cin;
    a.stride = sign > 0 ? l.stride : 1;
    a.sign = sign;
    return a;
}

// I rows = input rows x W^T for spiking layer i over `rows` timestep rows.
static skipper_status gemm_forward(skipper_ctx *c, int i, const uint16_t *in, float *I, int rows, int splits = -1) {
    Layer &l = c->L[i];
    const int fsp = splits > 0 ? splits : l.fsplit;
    if (rows <= 0) return SKIPPER_OK;
    sk::GemmLaunch g;
    const int nb = rows * c->B;
    bool ok;
    if (i == 0 && c->in_kind == 1)  // im2col rows [nb*H*W][K0] x padded weights [cout][K0]
        ok = get_plan(c, {0, in, l.wbp, I, (long long)nb * l.H * l.W, l.Cout, c->K0, 0, 0, 1}, g,
                      [&](sk::GemmLaunch *p) { return sk::plan_fc(p, in, l.wbp, I, nb * l.H * l.W, l.Cout, c->K0); });
    else if (l.icol && l.fwd_g) {  // narrow conv, cp.async gather producer
        const double M = (double)nb * l.H * l.W;
        ProfScope ps(c, K_GEMM_FWD, (double)nb * l.Nin * 2 + (double)l.wcount * 2 + (double)nb * l.N * 4,
                     2.0 * M * l.Cout * 9 * l.Cin);
        CK(sk::launch_conv_narrow(narrow_args(l, in, l.wb, I, nb, +1), c->st, c->num_sms));
        return SKIPPER_OK;
    } else if (l.icol && l.fwd_s)  // strided / narrow implicit conv: per-tap TMA boxes, no column buffer
        ok = get_plan(c, {7, in, l.wb, I, nb, l.Cin, l.Cout, l.H, l.W, l.stride}, g, [&](sk::GemmLaunch *p) {
            return sk::plan_conv_s(p, in, l.wb, I, nb, l.H, l.W, l.Cin, l.Cout, +1, l.stride);
        });
    else if (l.icol) {  // explicit im2col rows [nb*H*W][9*Cin] x weights [cout][9*Cin], in sample-row chunks
        const long long ch = icol_chunk(c);
        const int K = 9 * l.Cin;
        for (long long n0 = 0; n0 < nb; n0 += ch) {
            const int nbc = (int)std::min<long long>(ch, nb - n0);
            {
                ProfScope ps(c, K_IM2COL, (double)nbc * (l.Nin * 2 + (double)l.H * l.W * K * 2), 0);
                CK(sk::launch_im2col_bf16(in + n0 * l.Nin, c->cols[0], nbc, l.Hin, l.Win, l.Cin, l.H, l.W, l.stride,
                                          c->st));
            }
            const int M = nbc * l.H * l.W;
            float *Ic = I + n0 * l.N;
            ok = get_plan(c, {4, c->cols[0], l.wb, Ic, M, l.Cout, K, 0, 0, 1}, g,
                          [&](sk::GemmLaunch *p) { return sk::plan_fc(p, c->cols[0], l.wb, Ic, M, l.Cout, K); });
            const double Mf = M;
            CKS(run_gemm(c, g, ok, "forward", i, K_GEMM_FWD, Mf * K * 2 + (double)l.wcount * 2 + (double)nbc * l.N * 4,
                         2.0 * Mf * l.Cout * K));
        }
        return SKIPPER_OK;
    } else if (l.conv)
        ok = get_plan(c, {1, in, l.wb, I, nb, l.Cin, l.Cout, l.H, l.W, 1}, g, [&](sk::GemmLaunch *p) {
            return sk::plan_conv(p, in, l.wb, I, nb, l.H, l.W, l.Cin, l.Cout, +1);
        });
    else
        ok = get_plan(c, {0, in, l.wb, I, nb, l.Cout, l.Cin, 0, 0, fsp}, g, [&](sk::GemmLaunch *p) {
            return sk::plan_fc(p, in, l.wb, I, nb, l.Cout, l.Cin, fsp);
        });
    if (ok && g.d.splits != (l.fc ? fsp : 1)) return fail(c, SKIPPER_EUNSUPPORTED, "layer %d: split mismatch", i);
    const double M = (double)nb * l.H * l.W, K = (double)l.Cin * (l.conv ? 9 : 1);
    const double bytes = (double)nb * l.Nin * 2 + (double)l.wcount * 2 +
                         (double)nb * l.N * 4 * (l.fc ? fsp : 1);
    return run_gemm(c, g, ok, "forward", i, K_GEMM_FWD, bytes, 2.0 * M * l.Cout * K);
}

// ------------------------------------------------------------------------------------ step pieces
// SAM partial counters of one layer group (0 = input spikes, l + 1 = spiking layer l): [T][32]
static unsigned *spart(skipper_ctx *c, int group) { return c->s_part + (size_t)group * c->T * 32; }

static skipper_status begin_step(skipper_ctx *c, const unsigned char *x) {
    if (c->prof_on) prof_resolve(c);
    CKS(zero_dev(c, c->s_part, (size_t)(c->Ls + 1) * c->T * 32 * 4));
    if (c->u2_part) CKS(zero_dev(c, c->u2_part, (size_t)c->T * 32 * 8));
    CKS(zero_dev(c, c->cnt, (size_t)c->B * c->L[c->Ls - 1].Nout * 4));
    CKS(zero_dev(c, c->cnt_kept, (size_t)c->B * c->L[c->Ls - 1].Nout * 4));
    CKS(zero_dev(c, c->loss_dev, 4));
    CKS(zero_dev(c, c->dw_all, c->dw_total * 4));
    for (int i = 0; i < c->Ls; ++i) {
        Layer &l = c->L[i];
        const size_t bn = (size_t)c->B * l.N;
        CKS(zero_dev(c, l.U_run, l.sbn * 4));
        CKS(zero_dev(c, l.o_run, l.sbn));
        CKS(zero_dev(c, l.carry, bn * 4));
        if (c->cfg.debug_record)
            for (int k = 0; k < 2; ++k) {
                CKS(zero_dev(c, l.dbg[k], bn * c->T * 4));
                CKS(zero_dev(c, l.dbgo[k], bn * c->T));
            }
    }
    if (c->L[0].dwp) CKS(zero_dev(c, c->L[0].dwp, (size_t)c->L[0].Cout * c->K0 * 4));
    // the split-K weight-gradient slices the previous step summed: cleared on the weight-gradient stream, in
    // order after that step's reduction and before this step's first weight gradient, while the first pass
    // runs on the main stream (the reduction at the end of the step, on the critical path, only reads them)
    {
        cudaStream_t ws = c->prof_on ? c->st : c->st2;
        if (ws != c->st) {  // after everything the previous step issued on the main stream (its reduction
                            // ran there when it was profiled)
            CK(cudaEventRecord(c->ev_ready[0], c->st));
            CK(cudaStreamWaitEvent(ws, c->ev_ready[0], 0));
        }
        for (auto &l : c->L)
            if (l.dws) CK(cudaMemsetAsync(l.dws, 0, (size_t)l.wsl * l.wg_count * 4, ws));
    }
    c->x_cur = x;
    c->grads_ready = false;
    return SKIPPER_OK;
}

// Algorithmic HBM bytes of one scan launch: every operand read or written once.
static double scan_fwd_bytes(const skipper_ctx *c, const Layer &l, const sk::ScanFwdArgs &a) {
    const double rows = a.R, comp = a.R - (a.restore ? 1 : 0), bn = (double)c->B * l.N, bno = (double)c->B * l.Nout;
    double b = rows * bno * 2;                                        // layer output (bf16)
    b += a.I ? comp * bn * 4 : comp * (double)c->B * l.H * l.W * 4;  // currents, or input bit masks
    if (a.U_out) b += rows * bn * 4;                                  // stored membranes
    b += bn * 5 * (a.restore ? 1 : 2);                                // state / checkpoint in (and out)
    if (a.ckU) b += bn * 5;
    return b;
}
static double scan_bwd_bytes(const skipper_ctx *c, const Layer &l, const sk::ScanBwdArgs &a) {
    const double rows = a.R, bn = (double)c->B * l.N, bno = (double)c->B * l.Nout;
    double b = rows * bn * 4;                                         // U
    b += a.g_broadcast ? bno * 4 : rows * bno * 4;                    // g (pooled resolution when pooled)
    if (a.delta) b += rows * bn * 2;                                  // delta (bf16)
    b += bn * 8;                                                      // carry in/out
    return b;
}

// Layer-0 operand rows for R timesteps (t0 + r, or the device list `rows`) into c->xg.
static skipper_status stage_input(skipper_ctx *c, const int *rows, int t0, int R, bool sam) {
    const int kind = c->in_kind == 1 ? 1 : 0;
    const double bytes = (double)R * c->B * (c->in_elems + c->in_row * 2);
    ProfScope ps(c, K_STAGE, bytes, 0);
    const Layer &f = c->L[0];
    CK(sk::launch_stage_rows(c->x_cur, c->xg, rows, t0, R, c->B, kind == 1 ? f.H : c->in_h, kind == 1 ? f.W : c->in_w,
                             c->in_c, kind, c->K0, c->in_elems, sam ? spart(c, 0) : nullptr, c->st, f.stride));
    return SKIPPER_OK;
}

// Residual shortcut of layer i (reading 8): the source layer's bf16 output rows, same row order.
static void set_res_fwd(const skipper_ctx *c, int i, sk::ScanFwdArgs &a, const uint16_t *src_rows) {
    const Layer &l = c->L[i];
    if (l.res < 0) return;
    const Layer &src = c->L[l.res];
    a.res = src_rows;
    a.res_H = src.H;
    a.res_W = src.W;
    a.res_C = src.Cout;
    a.res_stride = src.H / l.H;
    a.res_lo = (l.Cout - src.Cout) / 2;
}

// First pass of the fc tail over segments g0 .. g0+nseg-1 (layer-major): GEMM with M = nseg*S*B, one scan
// per layer; tail_in holds the chunk's input rows (written by the last conv layer, or staged here).
static skipper_status forward_tail_chunk(skipper_ctx *c, int g0, int nseg) {
    if (c->tail0 >= c->Ls) return SKIPPER_OK;
    const int R = nseg * c->S, t0 = g0 * c->S;
    if (c->tail0 == 0) {
        uint16_t *save = c->xg;
        c->xg = c->tail_in;
        skipper_status st = stage_input(c, nullptr, t0, R, true);
        c->xg = save;
        CKS(st);
    }
    for (int i = c->tail0; i < c->Ls; ++i) {
        Layer &l = c->L[i];
        const size_t bn = (size_t)c->B * l.N;
        const uint16_t *in = i == c->tail0 ? c->tail_in : c->tailP[(i - c->tail0 - 1) & 1];
        uint16_t *out = c->tailP[(i - c->tail0) & 1];
        CKS(gemm_forward(c, i, in, c->tail_I, R, l.fsplitT));
        sk::ScanFwdArgs a{};
        a.I = c->tail_I;
        a.nsplit = l.fsplitT;
        a.split_stride = (long long)R * c->B * l.N;
        a.R = R;
        a.U_state = l.U_run;
        a.o_state = l.o_run;
        a.Po_out = out;
        a.ckU = l.ckU + (size_t)g0 * bn;
        a.cko = l.cko + (size_t)g0 * bn;
        a.ck_every = c->S;
        a.s_part = spart(c, i + 1);
        a.u2_part = c->u2_part;
        a.t0 = t0;
        a.cnt = (i == c->Ls - 1) ? c->cnt : nullptr;
        a.dbg_U = c->cfg.debug_record ? l.dbg[0] : nullptr;
        a.dbg_o = c->cfg.debug_record ? l.dbgo[0] : nullptr;
        a.B = c->B;
        a.H = l.H;
        a.W = l.W;
        a.C = l.Cout;
        a.pool = l.pool ? 1 : 0;
        a.lam = l.d.lambda;
        a.theta = l.d.theta;
        ProfScope ps(c, K_SCAN_FWD, scan_fwd_bytes(c, l, a), 0);
        CK(sk::launch_lif_fwd(a, c->st));
    }
    return SKIPPER_OK;
}

// Layer 0 as one fused kernel: im2col in smem, tcgen05, LIF, pooling, SAM, checkpoint (layer0.cu).
static skipper_status layer0_fused(skipper_ctx *c, int seg, int R, int t0, const int *row_t, bool restore,
                                   bool record, uint16_t *out) {
    Layer &l = c->L[0];
    const size_t bn = (size_t)c->B * l.N;
    sk::L0FwdArgs a{};
    a.x = c->x_cur;
    a.T = c->T;
    a.B = c->B;
    a.H = l.H;
    a.W = l.W;
    a.C0 = l.Cin;
    a.row_t = row_t;
    a.t0 = t0;
    a.R = R;
    a.restore = restore ? 1 : 0;
    a.wbp = l.wbp;
    a.N = l.Cout;
    a.pool = l.pool ? 1 : 0;
    a.lam = l.d.lambda;
    a.theta = l.d.theta;
    a.state_tm = 1;  // running state and checkpoints in the kernel's coalesced thread-major layout
    a.U_state = restore ? l.ckU + (size_t)seg * l.sbn : l.U_run;
    a.o_state = restore ? l.cko + (size_t)seg * l.sbn : l.o_run;
    a.U_out = (restore || record) ? l.Useg : nullptr;
    a.Po_out = out;
    a.ckU = (!restore && !record) ? l.ckU + (size_t)seg * l.sbn : nullptr;
    a.cko = (!restore && !record) ? l.cko + (size_t)seg * l.sbn : nullptr;
    a.ck_every = (a.ckU && R > c->S) ? c->S : 0;  // several segments per launch: a checkpoint every S rows
    a.ck_stride = (long long)l.sbn;
    a.s_part = restore ? nullptr : spart(c, 1);
    a.s_part_in = restore ? nullptr : spart(c, 0);
    a.u2_part = restore ? nullptr : c->u2_part;
    a.dbg_U = c->cfg.debug_record ? l.dbg[restore ? 1 : 0] : nullptr;
    a.dbg_o = c->cfg.debug_record ? l.dbgo[restore ? 1 : 0] : nullptr;
    // stored passes also emit the im2col rows the layer-0 weight gradient reads (no staging kernel)
    a.xg_out = (restore || record) && !c->l0_bwd_fused ? c->xg : nullptr;
    const double bytes = (double)R * c->B * (c->in_elems + l.Nout * 2 + (a.U_out ? l.N * 4 : 0) +
                                             (a.xg_out ? (double)l.H * l.W * c->K0 * 2 : 0)) + bn * 10;
    const double flops = 2.0 * R * c->B * l.H * l.W * l.Cout * 9 * l.Cin;
    ProfScope ps(c, K_L0_FWD, bytes, flops);
    CK(sk::launch_layer0_fwd(a, c->st, c->num_sms));
    return SKIPPER_OK;
}

// Conv layer i >= 1 as one kernel: tcgen05 implicit GEMM + LIF epilogue (conv_lif.cu).
static skipper_status conv_lif_rows(skipper_ctx *c, int i, int seg, const uint16_t *in, int R, int t0,
                                    const int *row_t, bool restore, bool record, uint16_t *out) {
    Layer &l = c->L[i];
    const size_t bn = (size_t)c->B * l.N;
    sk::ConvLifArgs a{};
    a.B = c->B;
    a.H = l.H;
    a.W = l.W;
    a.Cin = l.Cin;
    a.Cout = l.Cout;
    a.pool = l.pool ? 1 : 0;
    a.R = R;
    a.restore = restore ? 1 : 0;
    a.t0 = t0;
    a.row_t = row_t;
    a.state_tm = 1;  // running state and checkpoints in the kernel's coalesced thread-major layout
    a.U_state = restore ? l.ckU + (size_t)seg * l.sbn : l.U_run;
    a.o_state = restore ? l.cko + (size_t)seg * l.sbn : l.o_run;
    a.U_out = (restore || record) ? l.Useg : nullptr;
    a.Po_out = out;
    a.ckU = (!restore && !record) ? l.ckU + (size_t)seg * l.sbn : nullptr;
    a.cko = (!restore && !record) ? l.cko + (size_t)seg * l.sbn : nullptr;
    a.ck_every = (a.ckU && R > c->S) ? c->S : 0;
    a.ck_stride = (long long)l.sbn;
    a.s_part = restore ? nullptr : spart(c, i + 1);
    a.u2_part = restore ? nullptr : c->u2_part;
    a.dbg_U = c->cfg.debug_record ? l.dbg[restore ? 1 : 0] : nullptr;
    a.dbg_o = c->cfg.debug_record ? l.dbgo[restore ? 1 : 0] : nullptr;
    a.lam = l.d.lambda;
    a.theta = l.d.theta;
    const double comp = R - (restore ? 1 : 0);
    double bytes = comp * c->B * l.Nin * 2 + (double)l.wcount * 2 + (double)R * c->B * l.Nout * 2 + bn * 10;
    if (a.U_out) bytes += (double)R * bn * 4;
    if (a.ckU) bytes += bn * 5;
    const double flops = 2.0 * comp * c->B * l.H * l.W * l.Cout * 9.0 * l.Cin;
    ProfScope ps(c, K_CONV_LIF, bytes, flops);
    CK(sk::launch_conv_lif(in, R, l.wb, a, c->st, c->num_sms));
    return SKIPPER_OK;
}

// Narrow conv layer i as one kernel: cp.async gather conv on tcgen05 + the LIF scan in its epilogue.
static skipper_status narrow_lif_rows(skipper_ctx *c, int i, int seg, const uint16_t *in, int R, int t0,
                                      const int *row_t, bool restore, bool record, uint16_t *out) {
    Layer &l = c->L[i];
    const size_t bn = (size_t)c->B * l.N;
    sk::NarrowConvArgs a = narrow_args(l, in, l.wb, nullptr, c->B, +1);
    a.R = R;
    a.restore = restore ? 1 : 0;
    a.t0 = t0;
    a.row_t = row_t;
    a.U_state = restore ? l.ckU + (size_t)seg * bn : l.U_run;
    a.o_state = restore ? l.cko + (size_t)seg * bn : l.o_run;
    a.U_out = (restore || record) ? l.Useg : nullptr;
    a.Po_out = out;
    a.ckU = (!restore && !record) ? l.ckU + (size_t)seg * bn : nullptr;
    a.cko = (!restore && !record) ? l.cko + (size_t)seg * bn : nullptr;
    a.ck_every = (a.ckU && R > c->S) ? c->S : 0;
    a.ck_stride = (long long)bn;
    a.s_part = restore ? nullptr : spart(c, i + 1);
    a.u2_part = restore ? nullptr : c->u2_part;
    a.cnt = (i == c->Ls - 1) ? (restore ? c->cnt_kept : c->cnt) : nullptr;
    a.dbg_U = c->cfg.debug_record ? l.dbg[restore ? 1 : 0] : nullptr;
    a.dbg_o = c->cfg.debug_record ? l.dbgo[restore ? 1 : 0] : nullptr;
    a.lam = l.d.lambda;
    a.theta = l.d.theta;
    if (l.res >= 0) {
        const Layer &src = c->L[l.res];
        a.res = (restore || record) ? src.Po : c->P2[l.res % c->nP];
        a.res_H = src.H;
        a.res_W = src.W;
        a.res_C = src.Cout;
        a.res_stride = src.H / l.H;
        a.res_lo = (l.Cout - src.Cout) / 2;
    }
    const double comp = R - (restore ? 1 : 0);
    double bytes = comp * c->B * l.Nin * 2 + (double)l.wcount * 2 + (double)R * bn * 2 + bn * 10;
    if (a.U_out) bytes += (double)R * bn * 4;
    if (a.res) bytes += comp * c->B * c->L[l.res].N * 2;
    ProfScope ps(c, K_CONV_LIF, bytes, 2.0 * comp * c->B * l.H * l.W * l.Cout * 9.0 * l.Cin);
    static const bool nl_off = getenv("SKIPPER_NO_NARROW_LIF_MMA") && atoi(getenv("SKIPPER_NO_NARROW_LIF_MMA"));
    if (!nl_off && sk::narrow_lif_mma_supported(a.Cin, a.Cout, a.stride, a.H, a.W))
        CK(sk::launch_narrow_lif_mma(a, c->st, c->num_sms));
    else
        CK(sk::launch_conv_narrow_lif(a, c->st, c->num_sms));
    return SKIPPER_OK;
}

// Forward through all spiking layers for R rows starting at absolute time t0 (FIRST / RECORD).
static skipper_status forward_rows_first(skipper_ctx *c, int seg, int R, int t0, bool record) {
    // the staged layer-0 operand is needed by the first pass unless layer 0 is fused (or part of the
    // whole-sequence fc tail), and by the layer-0 weight gradient of FULL mode
    const int iend = record ? c->Ls : c->tail0;
    if ((record && !c->l0_bwd_fused && !c->l0_fused) || (iend > 0 && !c->l0_fused))
        CKS(stage_input(c, nullptr, t0, R, !c->l0_fused));
    for (int i = 0; i < iend; ++i) {
        Layer &l = c->L[i];
        const uint16_t *in;
        uint16_t *out;
        if (record) {
            in = i == 0 ? c->xg : c->L[i - 1].Po;
            out = l.Po;
        } else {
            in = i == 0 ? c->xg : c->P2[(i - 1) % c->nP];
            out = (i == c->tail0 - 1 && c->tail0 < c->Ls)
                      ? c->tail_in + (size_t)(seg % c->tail_G) * c->S * c->B * l.Nout  // row in the tail chunk
                      : c->P2[i % c->nP];
        }
        if (i == 0 && c->l0_fused) {
            CKS(layer0_fused(c, seg, R, t0, nullptr, false, record, out));
            continue;
        }
        if (l.cfused) {
            CKS(conv_lif_rows(c, i, seg, in, R, t0, nullptr, false, record, out));
            continue;
        }
        if (l.nlif) {
            CKS(narrow_lif_rows(c, i, seg, in, R, t0, nullptr, false, record, out));
            continue;
        }
        CKS(gemm_forward(c, i, in, c->I_buf, R));
        sk::ScanFwdArgs a{};
        a.I = c->I_buf;
        a.nsplit = l.fsplit;
        a.split_stride = (long long)R * c->B * l.N;
        a.R = R;
        a.restore = 0;
        a.U_state = l.U_run;
        a.o_state = l.o_run;
        a.U_out = record ? l.Useg : nullptr;
        a.Po_out = out;
        a.ckU = record ? nullptr : l.ckU + (size_t)seg * c->B * l.N;
        a.cko = record ? nullptr : l.cko + (size_t)seg * c->B * l.N;
        a.ck_every = (!record && R > c->S) ? c->S : 0;  // slots r / S, B*N apart
        a.s_part = spart(c, i + 1);
        a.u2_part = c->u2_part;
        a.row_t = nullptr;
        a.t0 = t0;
        a.cnt = (i == c->Ls - 1) ? c->cnt : nullptr;
        a.dbg_U = c->cfg.debug_record ? l.dbg[0] : nullptr;
        a.dbg_o = c->cfg.debug_record ? l.dbgo[0] : nullptr;
        a.B = c->B;
        a.H = l.H;
        a.W = l.W;
        a.C = l.Cout;
        a.pool = l.pool ? 1 : 0;
        a.lam = l.d.lambda;
        a.theta = l.d.theta;
        if (l.res >= 0) set_res_fwd(c, i, a, record ? c->L[l.res].Po : c->P2[l.res % c->nP]);
        {
            ProfScope ps(c, K_SCAN_FWD, scan_fwd_bytes(c, l, a), 0);
            CK(sk::launch_lif_fwd(a, c->st));
        }
    }
    return SKIPPER_OK;
}

static skipper_status comm_allreduce_s(skipper_ctx *c) {
    if (c->comm.comm) {
        std::string e;
        if (!c->comm.allreduce_i64(c->s_dev, (c->Ls + 1) * c->T, c->st, &e))  // per-layer counts
            return fail(c, SKIPPER_ENCCL, "%s", e.c_str());
    }
    return SKIPPER_OK;
}

// After the last FIRST segment: loss, SAM totals, SST and keep lists (Eq.4, Eq.5).
// Readout integrator + cross-entropy of cnt (normalised by 1/Tn): z, dz, loss += CE / B_global, and
// dL/da^{L-1} into g_last (through the GAP when the readout has one).
static skipper_status readout_forward(skipper_ctx *c, const int *labels, float invTn) {
    const Layer &last = c->L[c->Ls - 1];
    const Layer &ro = c->L.back();
    ProfScope ps1(c, K_READOUT, (double)c->B * last.Nout * 8 + (double)ro.wcount * 2, 4.0 * c->B * last.Nout * ro.Cout);
    c->launches += 2;  // z, cross-entropy and dL/da^{L-1} kernels
    if (ro.gap) {  // readout of the global average pool (reading 23); dL/da^{L-1} spread back over the positions
        const int P = (int)(last.Nout / last.Cout);
        c->launches += 2;
        CK(sk::launch_gap_reduce(c->cnt, c->cnt_gap, c->B, P, last.Cout, c->st));
        CK(sk::launch_readout_loss(ro.wb, c->cnt_gap, labels, c->z, c->dz, c->loss_dev, c->g_gap, c->B, ro.Cin,
                                   ro.Cout, invTn, 1.0f / c->Bg, c->st));
        CK(sk::launch_gap_expand(c->g_gap, c->g_last, c->B, P, last.Cout, c->st));
    } else {
        CK(sk::launch_readout_loss(ro.wb, c->cnt, labels, c->z, c->dz, c->loss_dev, c->g_last, c->B, (int)last.Nout,
                                   ro.Cout, invTn, 1.0f / c->Bg, c->st));
    }
    return SKIPPER_OK;
}

static skipper_status finish_first(skipper_ctx *c, const int *labels) {
    {
        ProfScope ps0(c, K_READOUT, (double)(c->Ls + 1) * c->T * 32 * 4, 0);
        CK(sk::launch_sam_finalize(c->s_part, c->s_dev, (c->Ls + 1) * c->T, c->st));
    }
    if (c->u2_part) {
        {
            ProfScope ps(c, K_READOUT, (double)c->T * 32 * 8 + (double)c->T * 8, 0);
            CK(sk::launch_sum32_f64(c->u2_part, c->u2_dev, c->T, c->st));
        }
        if (c->comm.comm) {
            std::string e;
            if (!c->comm.allreduce_f64(c->u2_dev, c->T, c->st, &e)) return fail(c, SKIPPER_ENCCL, "%s", e.c_str());
        }
        c->u2_host.assign(c->T, 0.0);
        CK(cudaMemcpyAsync(c->u2_host.data(), c->u2_dev, (size_t)c->T * 8, cudaMemcpyDeviceToHost, c->st));
    }
    if (c->cfg.mode != SKIPPER_MODE_TBPTT) CKS(readout_forward(c, labels, 1.0f / c->T));
    CKS(comm_allreduce_s(c));
    CK(cudaMemcpyAsync(c->counts_host.data(), c->s_dev, (size_t)(c->Ls + 1) * c->T * 8, cudaMemcpyDeviceToHost,
                       c->st));
    const double hs0 = c->host_prof ? now_ms() : 0.0;
    if (c->host_prof) {
        if (!c->hp_ev[0]) {
            cudaEventCreate(&c->hp_ev[0]);
            cudaEventCreate(&c->hp_ev[1]);
        }
        cudaEventRecord(c->hp_ev[0], c->st);
    }
    CK(cudaStreamSynchronize(c->st));  // the one host sync of the step
    if (c->host_prof) c->hp_sync += now_ms() - hs0;
    // SAM (Eq.4) and the policy metric: Eq.4 totals, or the neuron-count-weighted sum (reading 22)
    for (int t = 0; t < c->T; ++t) {
        long long tot = 0;
        double w = 0.0;
        for (int g = 0; g <= c->Ls; ++g) {
            const long long v = c->counts_host[(size_t)g * c->T + t];
            tot += v;
            w = w + (double)v / (double)(g == 0 ? c->in_elems : c->L[g - 1].N);
        }
        c->s_host[t] = tot;
        c->sam_host[t] = c->cfg.sam == SKIPPER_SAM_WEIGHTED ? w
                         : c->cfg.sam == SKIPPER_SAM_L2TRACE ? std::sqrt(c->u2_host[t]) : (double)tot;
    }
    const int C = c->C, S = c->S;
    c->kept.assign(C, {});
    c->keep.assign(c->T, 1);
    c->sst.assign(C, NAN);
    const bool skip = c->cfg.mode == SKIPPER_MODE_SKIP && c->cfg.p != 0.0;
    if (c->cfg.mode == SKIPPER_MODE_TBPTT) return SKIPPER_OK;  // no keep mask: the counts are for reporting
    for (int seg = 0; seg < C; ++seg) {
        if (skip)
            c->sst[seg] = c->cfg.sam != SKIPPER_SAM_SPIKES
                              ? sst_double(c->sam_host.data() + (size_t)seg * S, S, c->cfg.p)
                              : skipper_sst_host(c->s_host.data() + (size_t)seg * S, S, c->cfg.p);
        for (int t = seg * S; t < (seg + 1) * S; ++t) {
            bool k = true;
            if (skip && t != seg * S) k = c->sam_host[t] > c->sst[seg];
            c->keep[t] = k ? 1 : 0;
            if (k) c->kept[seg].push_back(t);
        }
    }
    c->kept_flat.assign((size_t)C * S, 0);
    c->Kmax = 0;
    for (int seg = 0; seg < C; ++seg) {
        std::copy(c->kept[seg].begin(), c->kept[seg].end(), c->kept_flat.begin() + (size_t)seg * S);
        c->Kmax = std::max<int>(c->Kmax, (int)c->kept[seg].size());
    }
    CK(cudaMemcpyAsync(c->kept_dev, c->kept_flat.data(), (size_t)C * S * 4, cudaMemcpyHostToDevice, c->st));
    // backward groups of G segments from the top: [C-G, C-1], [C-2G, C-G-1], ... (the lowest may be smaller)
    c->seg_lo.assign(C, 0);
    c->seg_off.assign(C, 0);
    c->grp_R.assign(C, 0);
    c->grp_start.assign(C, 0);
    c->grp_flat.clear();
    c->Rgrp = 0;
    for (int hi = C - 1; hi >= 0; hi -= c->G) {
        const int lo = std::max(0, hi - c->G + 1);
        c->grp_start[lo] = (int)c->grp_flat.size();
        int R = 0;
        for (int seg = lo; seg <= hi; ++seg) {
            c->seg_lo[seg] = lo;
            c->seg_off[seg] = R;
            R += (int)c->kept[seg].size();
            c->grp_flat.insert(c->grp_flat.end(), c->kept[seg].begin(), c->kept[seg].end());
        }
        c->grp_R[lo] = R;
        c->Rgrp = std::max(c->Rgrp, R);
    }
    if (c->G > 1)
        CK(cudaMemcpyAsync(c->grp_dev, c->grp_flat.data(), c->grp_flat.size() * 4, cudaMemcpyHostToDevice, c->st));
    return SKIPPER_OK;
}

static skipper_status recompute_segment_rows(skipper_ctx *c, int seg);

// RECOMPUTE of segment seg into rows seg_off[seg].. of its group's arena: the per-layer arena bases (stored
// membranes, layer outputs, layer-0 operand rows) are shifted for the duration of the segment
// ctx.wdb: point the layer outputs and the layer-0 operand rows at segment seg's slot
static void select_slot(skipper_ctx *c, int seg) {
    if (!c->wdb || !c->xgS[1]) return;
    const int s = seg & 1;
    for (auto &l : c->L) l.Po = l.PoS[s];
    c->xg = c->xgS[s];
    c->cur_slot = s;
}

static skipper_status recompute_segment(skipper_ctx *c, int seg) {
    if (c->wdb && c->xgS[1]) {
        select_slot(c, seg);
        // the weight gradients of segment seg + 2 read this slot's X operands
        if (c->slot_rec[c->cur_slot]) CK(cudaStreamWaitEvent(c->st, c->ev_slot[c->cur_slot], 0));
    }
    const size_t off = c->G > 1 ? (size_t)c->seg_off[seg] : 0;
    if (!off) return recompute_segment_rows(c, seg);
    for (auto &l : c->L) {
        if (l.readout) continue;
        l.Useg += off * c->B * l.N;
        l.Po += off * c->B * l.Nout;
    }
    c->xg += off * c->B * c->in_row;
    const skipper_status st = recompute_segment_rows(c, seg);
    for (auto &l : c->L) {
        if (l.readout) continue;
        l.Useg -= off * c->B * l.N;
        l.Po -= off * c->B * l.Nout;
    }
    c->xg -= off * c->B * c->in_row;
    return st;
}

static skipper_status recompute_segment_rows(skipper_ctx *c, int seg) {
    const int R = (int)c->kept[seg].size();
    const int *row_t = c->kept_dev + (size_t)seg * c->S;
    // layer-0 weight-gradient operand (written by the fused layer-0 kernel itself when it runs)
    if (!c->l0_bwd_fused && !c->l0_fused) CKS(stage_input(c, row_t, 0, R, false));
    for (int i = 0; i < c->Ls; ++i) {
        Layer &l = c->L[i];
        if (i == 0 && c->l0_fused) {
            CKS(layer0_fused(c, seg, R, 0, row_t, true, false, l.Po));
            continue;
        }
        const uint16_t *in = i == 0 ? c->xg : c->L[i - 1].Po;
        if (l.cfused) {
            CKS(conv_lif_rows(c, i, seg, in, R, 0, row_t, true, false, l.Po));
            continue;
        }
        if (l.nlif) {
            CKS(narrow_lif_rows(c, i, seg, in, R, 0, row_t, true, false, l.Po));
            continue;
        }
        const size_t in_row = (size_t)c->B * (i == 0 ? c->in_row : c->L[i - 1].Nout);
        if (R > 1)  // rows 1..R-1 (row 0 is the checkpoint)
            CKS(gemm_forward(c, i, in + in_row, c->I_buf + (size_t)c->B * l.N, R - 1));
        sk::ScanFwdArgs a{};
        a.I = c->I_buf;
        a.nsplit = l.fsplit;
        a.split_stride = (long long)(R - 1) * c->B * l.N;  // the GEMM covered rows 1..R-1
        a.R = R;
        a.restore = 1;
        a.U_state = l.ckU + (size_t)seg * c->B * l.N;
        a.o_state = l.cko + (size_t)seg * c->B * l.N;
        a.U_out = l.Useg;
        a.Po_out = l.Po;
        a.s_part = nullptr;
        a.row_t = row_t;
        a.cnt = (i == c->Ls - 1) ? c->cnt_kept : nullptr;
        a.dbg_U = c->cfg.debug_record ? l.dbg[1] : nullptr;
        a.dbg_o = c->cfg.debug_record ? l.dbgo[1] : nullptr;
        a.B = c->B;
        a.H = l.H;
        a.W = l.W;
        a.C = l.Cout;
        a.pool = l.pool ? 1 : 0;
        a.lam = l.d.lambda;
        a.theta = l.d.theta;
        if (l.res >= 0) set_res_fwd(c, i, a, c->L[l.res].Po);
        {
            ProfScope ps(c, K_SCAN_FWD, scan_fwd_bytes(c, l, a), 0);
            CK(sk::launch_lif_fwd(a, c->st));
        }
    }
    return SKIPPER_OK;
}

// Eq.2 backward over the R stored rows of a segment (layer-major, reverse t inside the scan).
static skipper_status join_wgrads(skipper_ctx *c) {
    for (int k = 0; k < 3; ++k)
        if (c->w_pending[k]) {
            CK(cudaStreamWaitEvent(c->st, c->ev_done[k], 0));
            c->w_pending[k] = false;
        }
    return SKIPPER_OK;
}

static long long rcv_neurons(const skipper_ctx *c, int i) { return i >= 0 ? c->L[i].N : 0; }

// Bucket plan for the overlapped dW allreduce: walking the spiking layers i = Ls-1 .. 1 (the order their
// final weight gradients appear in segment 0), close a bucket once it holds >= bucket_bytes; returns the
// 0/1 "closes a bucket" flags indexed by layer (layer 1 always closes the last one).
extern "C" int skipper_plan_buckets(const unsigned long long *wcount, int n_spiking, unsigned long long bucket_bytes,
                                    int *closes) {
    if (!wcount || !closes || n_spiking < 1) return -1;
    unsigned long long acc = 0;
    int nb = 0;
    for (int i = 0; i < n_spiking; ++i) closes[i] = 0;
    for (int i = n_spiking - 1; i >= 1; --i) {
        acc += wcount[i] * 4ULL;
        if (acc >= bucket_bytes || i == 1) {
            closes[i] = 1;
            acc = 0;
            ++nb;
        }
    }
    return nb;
}

// segment 0 only: layer i's weight gradient has been issued on `ws`; launch the bucket it closes
static skipper_status comm_after_wgrad(skipper_ctx *c, int i, cudaStream_t ws) {
    if (!c->comm.comm || i < 1 || !c->bucket_lo[i]) return SKIPPER_OK;
    int hi = i;
    while (hi + 1 < c->Ls && !c->bucket_lo[hi + 1]) ++hi;
    CK(cudaEventRecord(c->ev_w, ws));  // ws is in order: every wgrad of layers hi..i precedes this
    CK(cudaStreamWaitEvent(c->st3, c->ev_w, 0));
    const size_t cnt = (size_t)(c->L[hi].dw - c->L[i].dw) + c->L[hi].wcount;
    std::string e;
    if (!c->comm.allreduce_f32(c->L[i].dw, cnt, c->st3, &e)) return fail(c, SKIPPER_ENCCL, "%s", e.c_str());
    c->comm_pending = true;
    return SKIPPER_OK;
}

// segment 0 only: layer i's weight-gradient slices are final; sum them (slice order) into dW, on the stream
// that ran the weight gradients
static skipper_status reduce_wslices(skipper_ctx *c, int i, cudaStream_t ws) {
    Layer &l = c->L[i];
    if (!l.dws) return SKIPPER_OK;
    float *dst = (i == 0 && l.dwp) ? l.dwp : l.dw;
    ProfScope ps(c, K_GEMM_WGRAD, (double)l.wsl * l.wg_count * 4 + (double)l.wg_count * 8, 0, ws);
    CK(sk::launch_reduce_slices(l.dws, l.wsl, dst, l.wg_count, ws, 0));  // cleared by begin_step
    return SKIPPER_OK;
}

static skipper_status backward_rows(skipper_ctx *c, int R, const int *row_t, bool last_seg) {
    for (int i = c->Ls - 1; i >= 0; --i) {
        Layer &l = c->L[i];
        if (i == 0 && c->l0_bwd_fused) {  // reverse scan + weight gradient in one kernel, no delta in HBM
            sk::L0BwdArgs b{};
            b.x = c->x_cur;
            b.T = c->T;
            b.B = c->B;
            b.H = l.H;
            b.W = l.W;
            b.C0 = l.Cin;
            b.row_t = row_t;
            b.R = R;
            b.U = l.Useg;
            b.g = (c->Ls == 1) ? c->g_last : c->I_buf;
            b.carry = l.carry;
            b.dW = l.dwp;
            b.N = l.Cout;
            b.pool = l.pool ? 1 : 0;
            b.lam = l.d.lambda;
            b.theta = l.d.theta;
            b.surr = c->cfg.surrogate;
            b.gamma = c->cfg.surr_gamma;
            const double rows = (double)R * c->B;
            const double bytes = rows * (l.N * 4 + l.Nout * 4 + c->in_elems) + (double)c->B * l.N * 8;
            ProfScope ps(c, K_L0_BWD, bytes, 2.0 * rows * l.H * l.W * l.Cout * 9 * l.Cin);
            CK(sk::launch_layer0_bwd(b, c->st, c->num_sms));
            continue;
        }
        const int par = i % c->nD;
        uint16_t *dcur = c->d_buf2[par];
        if (c->w_pending[par]) {  // the wgrad of layer i+2 still reads this delta buffer
            CK(cudaStreamWaitEvent(c->st, c->ev_done[par], 0));
            c->w_pending[par] = false;
        }
        sk::ScanBwdArgs a{};
        a.g = (i == c->Ls - 1) ? c->g_last : c->I_buf;
        a.nsplit = (i == c->Ls - 1) ? 1 : c->L[i + 1].dsplit;  // dgrad of layer i+1 produced g
        a.split_stride = (long long)R * c->B * l.Nout;
        a.g_broadcast = (i == c->Ls - 1) ? 1 : 0;
        a.g_pooled = l.pool ? 1 : 0;
        a.U = l.Useg;
        a.carry = l.carry;
        a.delta = dcur;
        a.R = R;
        a.B = c->B;
        a.H = l.H;
        a.W = l.W;
        a.C = l.Cout;
        a.pool = l.pool ? 1 : 0;
        a.lam = l.d.lambda;
        a.theta = l.d.theta;
        a.surr = c->cfg.surrogate;
        a.gamma = c->cfg.surr_gamma;
        if (l.res_to >= 0) {  // shortcut source: S^T(delta of the receiving layer) joins g (reading 8)
            const Layer &rcv = c->L[l.res_to];
            a.res_delta = c->d_buf2[l.res_to % c->nD];
            a.res_C = rcv.Cout;
            a.res_stride = l.H / rcv.H;
            a.res_lo = (rcv.Cout - l.Cout) / 2;
        }
        if (!(i + 1 < c->Ls && c->L[i + 1].dlif)) {  // else delta_i came from layer i+1's fused dgrad
            double bytes = scan_bwd_bytes(c, l, a);
            if (a.res_delta) bytes += (double)R * c->B * rcv_neurons(c, l.res_to) * 2;
            ProfScope ps(c, K_SCAN_BWD, bytes, 0);
            CK(sk::launch_lif_bwd(a, c->st));
        }
        const int nb = R * c->B;
        const uint16_t *X = i == 0 ? c->xg : c->L[i - 1].Po;
        sk::GemmLaunch g;
        bool ok;
        const double Mw = (double)nb * l.H * l.W, Kw = (double)l.Cin * (l.conv ? 9 : 1);
        if (l.icol) {  // im2col of the layer input + weight-gradient GEMM per chunk, one column slot per delta slot
            cudaStream_t ws = c->prof_on ? c->st : c->st2;
            if (!c->prof_on) {
                CK(cudaEventRecord(c->ev_ready[par], c->st));
                CK(cudaStreamWaitEvent(c->st2, c->ev_ready[par], 0));
            }
            const long long ch = icol_chunk(c);
            static const bool nw_off = getenv("SKIPPER_NO_NARROW_WGRAD") && atoi(getenv("SKIPPER_NO_NARROW_WGRAD"));
            if (!nw_off && sk::narrow_wgrad_supported(l.Cin, l.Cout, l.stride, l.H, l.W)) {
                // no column buffer: the delta tile and the input rows it reads staged per CTA (narrow_wgrad.cu)
                const double M = (double)nb * l.H * l.W;
                ProfScope ps(c, K_GEMM_WGRAD, (double)nb * l.N * 2 + (double)nb * l.Nin * 2 + (double)l.wcount * 8,
                             2.0 * M * l.Cout * Kw, ws);
                CK(sk::launch_narrow_wgrad(X, dcur, l.dws ? l.dws : l.dw, nb, l.H, l.W, l.Cin, l.Cout, l.stride, ws,
                                           c->num_sms));
            }
            for (long long n0 = 0; n0 < nb && (nw_off || !sk::narrow_wgrad_supported(l.Cin, l.Cout, l.stride, l.H, l.W));
                 n0 += ch) {
                const int nbc = (int)std::min<long long>(ch, nb - n0);
                const int M = nbc * l.H * l.W;
                {
                    ProfScope ps(c, K_IM2COL, (double)nbc * l.Nin * 2 + (double)M * Kw * 2, 0, ws);
                    CK(sk::launch_im2col_bf16(X + n0 * l.Nin, c->cols[par], nbc, l.Hin, l.Win, l.Cin, l.H, l.W, l.stride,
                                              ws));
                }
                const uint16_t *Dc = dcur + n0 * l.N;
                float *dwo = l.dws ? l.dws : l.dw;
                ok = get_plan(c, {6, Dc, c->cols[par], dwo, M, l.Cout, (int)Kw, 0, 0, 0}, g, [&](sk::GemmLaunch *p) {
                    return sk::plan_fc_wgrad(p, Dc, c->cols[par], dwo, M, l.Cout, (int)Kw, c->num_sms, l.wsl);
                });
                CKS(run_gemm(c, g, ok, "wgrad", i, K_GEMM_WGRAD, (double)nbc * l.N * 2 + (double)M * Kw * 2 + (double)l.wcount * 8,
                             2.0 * M * l.Cout * Kw, ws));
            }
            if (last_seg) CKS(reduce_wslices(c, i, ws));
            if (!c->prof_on) {
                CK(cudaEventRecord(c->ev_done[par], c->st2));
                c->w_pending[par] = true;
            }
            if (last_seg) CKS(comm_after_wgrad(c, i, ws));
        } else if (i == 0 && c->in_kind == 1) {
            float *dwo = l.dws ? l.dws : l.dwp;
            ok = get_plan(c, {2, dcur, X, dwo, (long long)nb * l.H * l.W, l.Cout, c->K0, 0, 0, 0}, g,
                          [&](sk::GemmLaunch *p) {
                              return sk::plan_fc_wgrad(p, dcur, X, dwo, nb * l.H * l.W, l.Cout, c->K0, c->num_sms,
                                                       l.wsl);
                          });
        } else if (l.conv) {
            float *dwo = l.dws ? l.dws : l.dw;
            ok = get_plan(c, {3, dcur, X, dwo, nb, l.Cin, l.Cout, l.H, l.W, 0}, g, [&](sk::GemmLaunch *p) {
                return sk::plan_conv_wgrad(p, dcur, X, dwo, nb, l.H, l.W, l.Cin, l.Cout, c->num_sms, l.wsl);
            });
        } else {
            float *dwo = l.dws ? l.dws : l.dw;
            ok = get_plan(c, {2, dcur, X, dwo, nb, l.Cout, l.Cin, 0, 0, 0}, g, [&](sk::GemmLaunch *p) {
                return sk::plan_fc_wgrad(p, dcur, X, dwo, nb, l.Cout, l.Cin, c->num_sms, l.wsl);
            });
        }
        const double wbytes = (double)nb * l.N * 2 + (double)nb * l.Nin * 2 + (double)l.wcount * 8;
        if (l.icol) {
            // issued above
        } else if (c->prof_on) {  // profiling: serialise so each kernel's events bracket only itself
            CKS(run_gemm(c, g, ok, "wgrad", i, K_GEMM_WGRAD, wbytes, 2.0 * Mw * l.Cout * Kw));
            if (last_seg) CKS(reduce_wslices(c, i, c->st));
            if (last_seg) CKS(comm_after_wgrad(c, i, c->st));
        } else {   // weight gradient on the side stream, after this layer's delta is written
            CK(cudaEventRecord(c->ev_ready[par], c->st));
            CK(cudaStreamWaitEvent(c->st2, c->ev_ready[par], 0));
            CKS(run_gemm(c, g, ok, "wgrad", i, K_GEMM_WGRAD, wbytes, 2.0 * Mw * l.Cout * Kw, c->st2));
            if (last_seg) CKS(reduce_wslices(c, i, c->st2));
            CK(cudaEventRecord(c->ev_done[par], c->st2));
            c->w_pending[par] = true;
            if (last_seg) CKS(comm_after_wgrad(c, i, c->st2));
        }
        if (i > 0 && l.dlif) {  // g^{i-1} = conv(delta_i, flipped W_i) and layer i-1's reverse scan in one kernel
            Layer &pv = c->L[i - 1];
            const int ppar = (i - 1) % c->nD;
            if (c->w_pending[ppar]) {  // the wgrad of layer i+1 may still read layer i-1's delta buffer
                CK(cudaStreamWaitEvent(c->st, c->ev_done[ppar], 0));
                c->w_pending[ppar] = false;
            }
            sk::ConvLifArgs b{};
            b.B = c->B;
            b.H = l.H;
            b.W = l.W;
            b.Cin = l.Cout;
            b.Cout = l.Cin;
            b.R = R;
            b.lam = pv.d.lambda;
            b.theta = pv.d.theta;
            b.bU = pv.Useg;
            b.bcarry = pv.carry;
            b.bdelta = c->d_buf2[ppar];
            b.surr = c->cfg.surrogate;
            b.gamma = c->cfg.surr_gamma;
            const double M = (double)nb * l.H * l.W;
            ProfScope ps(c, K_DGRAD_LIF, (double)nb * l.N * 2 + (double)l.wcount * 2 + (double)nb * pv.N * (4 + 2) +
                         (double)c->B * pv.N * 8, 2.0 * M * l.Cin * 9 * l.Cout);
            CK(sk::launch_conv_lif_bwd(dcur, R, l.wt, b, c->st, c->num_sms));
        } else if (i > 0 && l.icol && l.dgrad_g) {  // stride 1: g = conv(delta, flipped W^T), cp.async gather kernel
            const double M = (double)nb * l.H * l.W;
            ProfScope ps(c, K_GEMM_DGRAD, (double)nb * l.N * 2 + (double)l.wcount * 2 + (double)nb * l.Nin * 4,
                         2.0 * M * l.Cin * 9 * l.Cout);
            static const bool nd_off = getenv("SKIPPER_NO_NARROW_DGRAD") && atoi(getenv("SKIPPER_NO_NARROW_DGRAD"));
            if (!nd_off && sk::narrow_dgrad_supported(l.Cin, l.Cout, l.H, l.W, 1))  // staged halo + ldmatrix gathers
                CK(sk::launch_narrow_dgrad(dcur, l.wt, c->I_buf, nb, l.H, l.W, l.Cin, l.Cout, 1, c->st, c->num_sms));
            else
                CK(sk::launch_conv_narrow(narrow_args(l, dcur, l.wt, c->I_buf, nb, -1), c->st, c->num_sms));
        } else if (i > 0 && l.icol && l.dgrad_s) {  // stride 1: g = conv(delta, flipped W^T) as a narrow implicit conv
            ok = get_plan(c, {8, dcur, l.wt, c->I_buf, nb, l.Cout, l.Cin, l.H, l.W, -1}, g, [&](sk::GemmLaunch *p) {
                return sk::plan_conv_s(p, dcur, l.wt, c->I_buf, nb, l.H, l.W, l.Cout, l.Cin, -1, 1);
            });
            const double M = (double)nb * l.H * l.W;
            CKS(run_gemm(c, g, ok, "dgrad", i, K_GEMM_DGRAD,
                         (double)nb * l.N * 2 + (double)l.wcount * 2 + (double)nb * l.Nin * 4, 2.0 * M * l.Cin * 9 * l.Cout));
        } else if (i > 0 && l.icol && !(getenv("SKIPPER_NO_NARROW_DGRAD") && atoi(getenv("SKIPPER_NO_NARROW_DGRAD"))) &&
                   sk::narrow_dgrad_supported(l.Cin, l.Cout, l.H, l.W, l.stride)) {  // strided: no column buffer
            const double M = (double)nb * l.H * l.W;
            ProfScope ps(c, K_GEMM_DGRAD, (double)nb * l.N * 2 + (double)l.wcount * 2 + (double)nb * l.Nin * 4,
                         2.0 * M * l.Cin * 9 * l.Cout);
            CK(sk::launch_narrow_dgrad(dcur, l.wt, c->I_buf, nb, l.H, l.W, l.Cin, l.Cout, l.stride, c->st, c->num_sms));
        } else if (i > 0 && l.icol) {  // per chunk: dcols = delta_i W_i (columns (ci, tap)), then the col2im gather into g
            const long long ch = icol_chunk(c);
            const int N = 9 * l.Cin;
            for (long long n0 = 0; n0 < nb; n0 += ch) {
                const int nbc = (int)std::min<long long>(ch, nb - n0);
                const int M = nbc * l.H * l.W;
                const uint16_t *Dc = dcur + n0 * l.N;
                ok = get_plan(c, {5, Dc, l.wt, c->dcols, M, N, l.Cout, 0, 0, 1}, g, [&](sk::GemmLaunch *p) {
                    return sk::plan_fc(p, Dc, l.wt, c->dcols, M, N, l.Cout);
                });
                const double bytes = (double)nbc * l.N * 2 + (double)l.wcount * 2 + (double)M * N * 4;
                CKS(run_gemm(c, g, ok, "dgrad", i, K_GEMM_DGRAD, bytes, 2.0 * M * N * l.Cout));
                ProfScope ps(c, K_IM2COL, (double)M * N * 4 + (double)nbc * l.Nin * 4, 0);
                CK(sk::launch_col2im_f32(c->dcols, c->I_buf + n0 * l.Nin, nbc, l.Hin, l.Win, l.Cin, l.H, l.W, l.stride,
                                         c->st));
            }
        } else if (i > 0) {  // g for layer i-1 = delta_i W_i  (gradient wrt its (pooled) output)
            if (l.conv)
                ok = get_plan(c, {1, dcur, l.wt, c->I_buf, nb, l.Cout, l.Cin, l.H, l.W, -1}, g,
                              [&](sk::GemmLaunch *p) {
                                  return sk::plan_conv(p, dcur, l.wt, c->I_buf, nb, l.H, l.W, l.Cout, l.Cin, -1);
                              });
            else
                ok = get_plan(c, {0, dcur, l.wt, c->I_buf, nb, l.Cin, l.Cout, 0, 0, l.dsplit}, g,
                              [&](sk::GemmLaunch *p) {
                                  return sk::plan_fc(p, dcur, l.wt, c->I_buf, nb, l.Cin, l.Cout, l.dsplit);
                              });
            const double M = (double)nb * l.H * l.W, K = (double)l.Cout * (l.conv ? 9 : 1);
            const double bytes = (double)nb * l.N * 2 + (double)l.wcount * 2 + (double)nb * l.Nin * 4 * l.dsplit;
            CKS(run_gemm(c, g, ok, "dgrad", i, K_GEMM_DGRAD, bytes, 2.0 * M * l.Cin * K));
        }
    }
    // the next segment reuses the arena (X operands, delta buffers): wait for the weight gradients - or, with
    // the two X slots (ctx.wdb), only mark this slot busy until they finish (the delta buffers keep their
    // per-buffer w_pending waits)
    if (c->wdb && c->xgS[1] && !last_seg && !c->prof_on) {
        CK(cudaEventRecord(c->ev_slot[c->cur_slot], c->st2));
        c->slot_rec[c->cur_slot] = true;
        return SKIPPER_OK;
    }
    return join_wgrads(c);
}

// ------------------------------------------------------------------------------------ TBPTT (NEXT-4)
// Window w of truncated BPTT (reading 24): forward from the running state storing U and the outputs of
// its t' = S rows, then the window's own readout and loss (added to the step loss).
static skipper_status tbptt_forward(skipper_ctx *c, int w, const int *labels) {
    CKS(zero_dev(c, c->cnt, (size_t)c->B * c->L[c->Ls - 1].Nout * 4));
    CKS(forward_rows_first(c, w, c->S, w * c->S, true));
    return readout_forward(c, labels, 1.0f / c->S);
}

// Backward of window w: the graph is cut at the window's end (zero carry), weight gradients accumulate.
static skipper_status tbptt_backward(skipper_ctx *c, int w) {
    for (int i = 0; i < c->Ls; ++i) CKS(zero_dev(c, c->L[i].carry, (size_t)c->B * c->L[i].N * 4));
    CKS(backward_rows(c, c->S, nullptr, w == c->C - 1));
    const Layer &last = c->L[c->Ls - 1];
    const Layer &ro = c->L.back();
    ProfScope ps(c, K_READOUT, (double)c->B * (last.Nout + ro.Cout) * 4 + (double)ro.wcount * 8,
                 2.0 * c->B * last.Nout * ro.Cout);
    const float *cin = c->cnt;
    int D = (int)last.Nout;
    if (ro.gap) {
        c->launches += 1;
        CK(sk::launch_gap_reduce(c->cnt, c->cnt_gap, c->B, (int)(last.Nout / last.Cout), last.Cout, c->st));
        cin = c->cnt_gap;
        D = ro.Cin;
    }
    CK(sk::launch_readout_wgrad(c->dz, cin, ro.dw, c->B, D, ro.Cout, 1.0f / c->S, c->st, 1));
    return SKIPPER_OK;
}

// After the last window: layer-0 unpad, the last dW buckets, SAM counts (reporting), debug copies.
static skipper_status tbptt_finish(skipper_ctx *c) {
    Layer &l0 = c->L[0];
    const Layer &ro = c->L.back();
    if (l0.dwp) {
        const int cols = (int)(l0.wcount / l0.Cout);
        ProfScope ps(c, K_UNPAD, (double)l0.Cout * (c->K0 + cols) * 4, 0);
        CK(sk::launch_unpad_f32(l0.dwp, l0.dw, l0.Cout, cols, c->K0, c->st));
    }
    if (c->comm.comm) {
        CK(cudaEventRecord(c->ev_w, c->st));
        CK(cudaStreamWaitEvent(c->st3, c->ev_w, 0));
        std::string e;
        if (!c->comm.allreduce_f32(l0.dw, l0.wcount, c->st3, &e) || !c->comm.allreduce_f32(ro.dw, ro.wcount, c->st3, &e))
            return fail(c, SKIPPER_ENCCL, "%s", e.c_str());
        c->comm_pending = true;
    }
    CKS(finish_first(c, nullptr));
    if (c->cfg.debug_record)
        for (int i = 0; i < c->Ls; ++i) {
            const size_t bn = (size_t)c->B * c->L[i].N * c->T;
            CK(cudaMemcpyAsync(c->L[i].dbg[1], c->L[i].dbg[0], bn * 4, cudaMemcpyDeviceToDevice, c->st));
            CK(cudaMemcpyAsync(c->L[i].dbgo[1], c->L[i].dbgo[0], bn, cudaMemcpyDeviceToDevice, c->st));
        }
    return SKIPPER_OK;
}

// ------------------------------------------------------------------------------------ public schedule
extern "C" skipper_status skipper_forward_segment(skipper_ctx *c, int seg, int pass, const unsigned char *x_dev,
                                                  const int *labels_dev) {
    CKS(check_ctx(c));
    if (!x_dev) return fail(c, SKIPPER_EINVAL, "null input");
    const bool full = c->cfg.mode == SKIPPER_MODE_FULL;
    if (pass == SKIPPER_PASS_RECORD) {
        if (!full || seg != 0) return fail(c, SKIPPER_EORDER, "RECORD is the single pass of FULL mode (seg 0)");
        if (!labels_dev) return fail(c, SKIPPER_EINVAL, "RECORD needs labels");
        CKS(begin_step(c, x_dev));
        CKS(arena_rows(c, c->T));
        CKS(forward_rows_first(c, 0, c->T, 0, true));
        CKS(finish_first(c, labels_dev));
        c->phase = PH_RECOMPUTED;
        c->next_seg = 0;
        return SKIPPER_OK;
    }
    if (full) return fail(c, SKIPPER_EORDER, "FULL mode uses the RECORD pass");
    if (c->cfg.mode == SKIPPER_MODE_TBPTT) {  // window w: forward + its loss (then backward_segment(w))
        if (pass != SKIPPER_PASS_FIRST) return fail(c, SKIPPER_EORDER, "TBPTT windows use the FIRST pass");
        if (!labels_dev) return fail(c, SKIPPER_EINVAL, "every TBPTT window needs labels");
        if (seg == 0) {
            if (c->phase != PH_IDLE && c->phase != PH_BWD_DONE)
                return fail(c, SKIPPER_EORDER, "FIRST(0) while an iteration is in flight");
            CKS(begin_step(c, x_dev));
            CKS(arena_rows(c, c->S));
            c->phase = PH_FIRST;
            c->next_seg = 0;
        }
        if (c->phase != PH_FIRST || seg != c->next_seg)
            return fail(c, SKIPPER_EORDER, "TBPTT windows run FIRST(w), BACKWARD(w) for w = 0..C-1 (expected %d)",
                        c->next_seg);
        if (x_dev != c->x_cur) return fail(c, SKIPPER_EINVAL, "x_dev changed within an iteration");
        CKS(tbptt_forward(c, seg, labels_dev));
        c->phase = PH_RECOMPUTED;
        return SKIPPER_OK;
    }
    if (pass == SKIPPER_PASS_FIRST) {
        if (seg == 0) {
            if (c->phase != PH_IDLE && c->phase != PH_BWD_DONE && c->phase != PH_FIRST)
                return fail(c, SKIPPER_EORDER, "FIRST(0) while an iteration is in flight");
            CKS(begin_step(c, x_dev));
            CKS(arena_first(c));
            c->phase = PH_FIRST;
            c->next_seg = 0;
        }
        if (c->phase != PH_FIRST || seg != c->next_seg)
            return fail(c, SKIPPER_EORDER, "FIRST segments must run 0..C-1 in order (expected %d)", c->next_seg);
        if (x_dev != c->x_cur) return fail(c, SKIPPER_EINVAL, "x_dev changed within an iteration");
        // checked before any work or state change, so a retry with labels can continue from here
        if (seg == c->C - 1 && !labels_dev) return fail(c, SKIPPER_EINVAL, "the last FIRST segment needs labels");
        if (seg == 0) c->fp_s0 = 0;
        const int end = first_chunk_end(c, c->fp_s0);
        if (seg + 1 == end) {  // the chunk's last segment: its layers before the tail run now, F segments at once
            CKS(forward_rows_first(c, c->fp_s0, (end - c->fp_s0) * c->S, c->fp_s0 * c->S, false));
            c->fp_s0 = end;
        }
        c->next_seg = seg + 1;
        if ((seg + 1) % c->tail_G == 0 || seg == c->C - 1)  // the fc tail of the chunk that ends here
            CKS(forward_tail_chunk(c, seg - seg % c->tail_G, seg % c->tail_G + 1));
        if (seg == c->C - 1) {
            CKS(finish_first(c, labels_dev));
            CKS(arena_rows(c, std::max(c->Kmax, c->Rgrp)));
            c->phase = PH_READY_BWD;
            c->next_seg = c->C - 1;
        }
        return SKIPPER_OK;
    }
    if (pass == SKIPPER_PASS_RECOMPUTE) {
        if (c->phase != PH_READY_BWD || seg != c->next_seg)
            return fail(c, SKIPPER_EORDER, "RECOMPUTE must follow FIRST / the previous BACKWARD (expected seg %d)",
                        c->next_seg);
        if (x_dev != c->x_cur) return fail(c, SKIPPER_EINVAL, "x_dev changed within an iteration");
        CKS(recompute_segment(c, seg));
        c->phase = PH_RECOMPUTED;
        return SKIPPER_OK;
    }
    return fail(c, SKIPPER_EINVAL, "unknown pass %d", pass);
}

extern "C" skipper_status skipper_backward_segment(skipper_ctx *c, int seg) {
    CKS(check_ctx(c));
    if (c->phase != PH_RECOMPUTED || seg != c->next_seg)
        return fail(c, SKIPPER_EORDER, "BACKWARD(%d) must follow RECOMPUTE(%d)", seg, c->next_seg);
    if (c->cfg.mode == SKIPPER_MODE_TBPTT) {
        CKS(tbptt_backward(c, seg));
        if (seg == c->C - 1) {
            CKS(tbptt_finish(c));
            c->phase = PH_BWD_DONE;
            c->grads_ready = true;
            CKS(arena_free(c));
        } else {
            c->phase = PH_FIRST;
            c->next_seg = seg + 1;
        }
        return SKIPPER_OK;
    }
    const bool full = c->cfg.mode == SKIPPER_MODE_FULL;
    if (!full && c->G > 1 && c->seg_lo[seg] != seg) {  // grouped: the group's backward runs at its lowest segment
        c->phase = PH_READY_BWD;
        c->next_seg = seg - 1;
        return SKIPPER_OK;
    }
    select_slot(c, seg);
    const int R = full ? c->T : c->G > 1 ? c->grp_R[seg] : (int)c->kept[seg].size();
    const int *row_t = full ? nullptr : c->G > 1 ? c->grp_dev + c->grp_start[seg] : c->kept_dev + (size_t)seg * c->S;
    CKS(backward_rows(c, R, row_t, seg == 0));
    if (seg == 0) {
        const Layer &last = c->L[c->Ls - 1];
        const Layer &ro = c->L.back();
        Layer &l0 = c->L[0];
        if (l0.dwp) {  // padded im2col weight gradient -> [cout][9*cin]
            const int cols = (int)(l0.wcount / l0.Cout);
            ProfScope ps(c, K_UNPAD, (double)l0.Cout * (c->K0 + cols) * 4, 0);
            CK(sk::launch_unpad_f32(l0.dwp, l0.dw, l0.Cout, cols, c->K0, c->st));
        }
        ProfScope ps(c, K_READOUT, (double)c->B * (last.Nout + ro.Cout) * 4 + (double)ro.wcount * 4,
                     2.0 * c->B * last.Nout * ro.Cout);
        const float *cin = full ? c->cnt : c->cnt_kept;
        int D = (int)last.Nout;
        if (ro.gap) {
            c->launches += 1;
            CK(sk::launch_gap_reduce(cin, c->cnt_gap, c->B, (int)(last.Nout / last.Cout), last.Cout, c->st));
            cin = c->cnt_gap;
            D = ro.Cin;
        }
        CK(sk::launch_readout_wgrad(c->dz, cin, ro.dw, c->B, D, ro.Cout, 1.0f / c->T, c->st));
        if (c->comm.comm) {  // the last buckets: layer 0 (final after the unpad above) and the readout
            CK(cudaEventRecord(c->ev_w, c->st));
            CK(cudaStreamWaitEvent(c->st3, c->ev_w, 0));
            std::string e;
            if (!c->comm.allreduce_f32(l0.dw, l0.wcount, c->st3, &e) ||
                !c->comm.allreduce_f32(ro.dw, ro.wcount, c->st3, &e))
                return fail(c, SKIPPER_ENCCL, "%s", e.c_str());
            c->comm_pending = true;
        }
        if (c->cfg.debug_record && full)
            for (int i = 0; i < c->Ls; ++i) {
                const size_t bn = (size_t)c->B * c->L[i].N * c->T;
                CK(cudaMemcpyAsync(c->L[i].dbg[1], c->L[i].dbg[0], bn * 4, cudaMemcpyDeviceToDevice, c->st));
                CK(cudaMemcpyAsync(c->L[i].dbgo[1], c->L[i].dbgo[0], bn, cudaMemcpyDeviceToDevice, c->st));
            }
        c->phase = PH_BWD_DONE;
        c->grads_ready = true;
        CKS(arena_free(c));
    } else {
        c->phase = PH_READY_BWD;
        c->next_seg = seg - 1;
    }
    return SKIPPER_OK;
}

extern "C" skipper_status skipper_optimizer_step(skipper_ctx *c) {
    CKS(check_ctx(c));
    if (c->phase != PH_BWD_DONE || !c->grads_ready)
        return fail(c, SKIPPER_EORDER, "optimizer_step needs a completed backward");
    if (c->comm_pending) {  // the bucketed dW allreduce issued during segment 0's backward
        CK(cudaEventRecord(c->ev_comm, c->st3));
        CK(cudaStreamWaitEvent(c->st, c->ev_comm, 0));
        c->comm_pending = false;
    }
    c->adam_step += 1;
    const double b1 = c->cfg.beta1, b2 = c->cfg.beta2;
    const float bc1 = (float)(1.0 - std::pow(b1, (double)c->adam_step));
    const float bc2s = (float)std::sqrt(1.0 - std::pow(b2, (double)c->adam_step));
    for (int i = 0; i < (int)c->L.size(); ++i) {
        Layer &l = c->L[i];
        {
            ProfScope ps(c, K_ADAM, (double)l.wcount * 26, 0);
            CK(sk::launch_adam(l.w, l.dw, l.m, l.v, l.wb, l.wcount, c->cfg.lr, c->cfg.beta1, c->cfg.beta2, c->cfg.eps,
                               bc1, bc2s, c->st));
        }
        if (l.wbp) {
            ProfScope ps(c, K_ADAM, (double)l.wcount * 6, 0);
            CK(sk::launch_cast_pad_bf16(l.w, l.wbp, l.Cout, (int)(l.wcount / l.Cout), c->K0, c->st));
        }
        if (l.wt) {
            ProfScope ps(c, K_ADAM, (double)l.wcount * 4, 0);
            if (l.conv)
                CK(sk::launch_transpose_bf16(l.wb, l.wt, l.Cout, 9, l.Cin, c->st));
            else
                CK(sk::launch_transpose_bf16(l.wb, l.wt, l.Cout, 1, l.Cin, c->st));
        }
    }
    c->grads_ready = false;
    c->phase = PH_IDLE;
    return SKIPPER_OK;
}

extern "C" skipper_status skipper_step(skipper_ctx *c, const unsigned char *x_dev, const int *labels_dev,
                                       float *loss_host) {
    CKS(check_ctx(c));
    if (!x_dev || !labels_dev) return fail(c, SKIPPER_EINVAL, "null input or labels");
    if (c->cfg.mode == SKIPPER_MODE_FULL) {
        CKS(skipper_forward_segment(c, 0, SKIPPER_PASS_RECORD, x_dev, labels_dev));
        CKS(skipper_backward_segment(c, 0));
    } else if (c->cfg.mode == SKIPPER_MODE_TBPTT) {
        c->phase = PH_IDLE;
        for (int w = 0; w < c->C; ++w) {
            CKS(skipper_forward_segment(c, w, SKIPPER_PASS_FIRST, x_dev, labels_dev));
            CKS(skipper_backward_segment(c, w));
        }
    } else {
        c->phase = PH_IDLE;
        const double h0 = c->host_prof ? now_ms() : 0.0;
        const double s0 = c->hp_sync;
        for (int seg = 0; seg < c->C; ++seg)
            CKS(skipper_forward_segment(c, seg, SKIPPER_PASS_FIRST, x_dev, seg == c->C - 1 ? labels_dev : nullptr));
        const double h1 = c->host_prof ? now_ms() : 0.0;
        if (c->host_prof && c->hp_ev[1]) cudaEventRecord(c->hp_ev[1], c->st);  // after the kept-list H2D copy
        for (int seg = c->C - 1; seg >= 0; --seg) {
            CKS(skipper_forward_segment(c, seg, SKIPPER_PASS_RECOMPUTE, x_dev, nullptr));
            CKS(skipper_backward_segment(c, seg));
        }
        if (c->host_prof) {
            c->hp_first += (h1 - h0) - (c->hp_sync - s0);
            c->hp_bwd += now_ms() - h1;
            c->hp_steps++;
            float gap = 0.f;
            if (c->hp_ev[1] && cudaEventSynchronize(c->hp_ev[1]) == cudaSuccess &&
                cudaEventElapsedTime(&gap, c->hp_ev[0], c->hp_ev[1]) == cudaSuccess)
                c->hp_gap += gap;
        }
    }
    CKS(skipper_optimizer_step(c));
    if (loss_host) {
        CK(cudaMemcpyAsync(loss_host, c->loss_dev, 4, cudaMemcpyDeviceToHost, c->st));
        CK(cudaStreamSynchronize(c->st));
    }
    return SKIPPER_OK;
}

extern "C" skipper_status skipper_step_host(skipper_ctx *c, const unsigned char *x_host, const int *labels_host,
                                            float *loss_host) {
    CKS(check_ctx(c));
    if (!x_host || !labels_host) return fail(c, SKIPPER_EINVAL, "null host input");
    const size_t xbytes = (size_t)c->T * c->B * c->in_elems;
    if (!c->x_stage) {
        CKS(alloc_arr(c, &c->x_stage, xbytes));
    }
    if (!c->y_stage) CKS(alloc_arr(c, &c->y_stage, (size_t)c->B));
    CK(cudaMemcpyAsync(c->x_stage, x_host, xbytes, cudaMemcpyHostToDevice, c->st));
    CK(cudaMemcpyAsync(c->y_stage, labels_host, (size_t)c->B * 4, cudaMemcpyHostToDevice, c->st));
    float loss = 0.f;
    CKS(skipper_step(c, c->x_stage, c->y_stage, &loss));
    if (loss_host) *loss_host = loss;
    return SKIPPER_OK;
}

// ------------------------------------------------------------------------------------ encoder (NEXT-3)
extern "C" skipper_status skipper_encode_poisson(const float *x_dev, const float *rates_dev, unsigned long long seed,
                                                 int T, int B, long long D, unsigned char *out_dev, void *stream) {
    if (!x_dev || !rates_dev || !out_dev || T < 0 || B < 0 || D < 0)
        return fail(nullptr, SKIPPER_EINVAL, "encode_poisson: bad arguments");
    const cudaError_t e = sk::launch_poisson_encode(x_dev, rates_dev, seed, T, B, D, out_dev, static_cast<cudaStream_t>(stream));
    if (e != cudaSuccess) return fail(nullptr, SKIPPER_ECUDA, "encode_poisson: %s", cudaGetErrorString(e));
    return SKIPPER_OK;
}

extern "C" skipper_status skipper_step_encoded(skipper_ctx *c, const float *x_dev, const float *rates_dev,
                                               unsigned long long seed, const int *labels_dev, float *loss_host) {
    CKS(check_ctx(c));
    if (!x_dev || !rates_dev || !labels_dev) return fail(c, SKIPPER_EINVAL, "null input");
    if (!c->x_enc) CKS(alloc_arr(c, &c->x_enc, (size_t)c->T * c->B * c->in_elems));
    {
        ProfScope ps(c, K_STAGE, (double)c->B * c->in_elems * 4 + (double)c->T * c->B * c->in_elems, 0);
        CK(sk::launch_poisson_encode(x_dev, rates_dev, seed, c->T, c->B, c->in_elems, c->x_enc, c->st));
    }
    return skipper_step(c, c->x_enc, labels_dev, loss_host);
}

extern "C" skipper_status skipper_step_host_encoded(skipper_ctx *c, const float *x_host, const float *rates_host,
                                                    unsigned long long seed, const int *labels_host, float *loss_host) {
    CKS(check_ctx(c));
    if (!x_host || !rates_host || !labels_host) return fail(c, SKIPPER_EINVAL, "null host input");
    if (!c->img_stage) {
        CKS(alloc_arr(c, &c->img_stage, (size_t)c->B * c->in_elems));
        CKS(alloc_arr(c, &c->rates_stage, (size_t)c->T));
    }
    if (!c->y_stage) CKS(alloc_arr(c, &c->y_stage, (size_t)c->B));
    CK(cudaMemcpyAsync(c->img_stage, x_host, (size_t)c->B * c->in_elems * 4, cudaMemcpyHostToDevice, c->st));
    CK(cudaMemcpyAsync(c->rates_stage, rates_host, (size_t)c->T * 4, cudaMemcpyHostToDevice, c->st));
    CK(cudaMemcpyAsync(c->y_stage, labels_host, (size_t)c->B * 4, cudaMemcpyHostToDevice, c->st));
    float loss = 0.f;
    CKS(skipper_step_encoded(c, c->img_stage, c->rates_stage, seed, c->y_stage, &loss));
    if (loss_host) *loss_host = loss;
    return SKIPPER_OK;
}

// ------------------------------------------------------------------------------------ introspection
extern "C" skipper_status skipper_get_loss(skipper_ctx *c, float *loss_host) {
    CKS(check_ctx(c));
    CK(cudaMemcpyAsync(loss_host, c->loss_dev, 4, cudaMemcpyDeviceToHost, c->st));
    CK(cudaStreamSynchronize(c->st));
    return SKIPPER_OK;
}
extern "C" skipper_status skipper_get_spike_sums(skipper_ctx *c, long long *s_host) {
    CKS(check_ctx(c));
    CK(cudaStreamSynchronize(c->st));
    std::copy(c->s_host.begin(), c->s_host.end(), s_host);
    return SKIPPER_OK;
}
extern "C" skipper_status skipper_get_keep_mask(skipper_ctx *c, unsigned char *keep_host) {
    CKS(check_ctx(c));
    std::copy(c->keep.begin(), c->keep.end(), keep_host);
    return SKIPPER_OK;
}
extern "C" skipper_status skipper_get_layer_spike_counts(skipper_ctx *c, long long *counts_host) {
    CKS(check_ctx(c));
    if (!counts_host) return fail(c, SKIPPER_EINVAL, "null output");
    std::copy(c->counts_host.begin(), c->counts_host.end(), counts_host);
    return SKIPPER_OK;
}
extern "C" skipper_status skipper_get_sam(skipper_ctx *c, double *sam_host) {
    CKS(check_ctx(c));
    if (!sam_host) return fail(c, SKIPPER_EINVAL, "null output");
    std::copy(c->sam_host.begin(), c->sam_host.end(), sam_host);
    return SKIPPER_OK;
}
extern "C" skipper_status skipper_get_sst(skipper_ctx *c, double *sst_host) {
    CKS(check_ctx(c));
    std::copy(c->sst.begin(), c->sst.end(), sst_host);
    return SKIPPER_OK;
}
extern "C" skipper_status skipper_mem_stats(skipper_ctx *c, size_t *cur, size_t *peak) {
    CKS(check_ctx(c));
    if (cur) *cur = c->cur_bytes;
    if (peak) *peak = c->peak_bytes;
    return SKIPPER_OK;
}
extern "C" skipper_status skipper_reset_peak(skipper_ctx *c) {
    CKS(check_ctx(c));
    c->peak_bytes = c->cur_bytes;
    return SKIPPER_OK;
}
extern "C" skipper_status skipper_debug_copy(skipper_ctx *c, int which, int layer, void *dst, size_t bytes) {
    CKS(check_ctx(c));
    if (!c->cfg.debug_record) return fail(c, SKIPPER_EINVAL, "debug_record is off");
    if (layer < 0 || layer >= c->Ls || which < 0 || which > 3 || !dst)
        return fail(c, SKIPPER_EINVAL, "bad debug request");
    const Layer &l = c->L[layer];
    const size_t n = (size_t)c->T * c->B * l.N;
    const bool isU = which == 0 || which == 2;
    const size_t need = n * (isU ? 4 : 1);
    if (bytes < need) return fail(c, SKIPPER_EINVAL, "debug buffer too small (%zu < %zu)", bytes, need);
    const void *src = isU ? (const void *)l.dbg[which / 2] : (const void *)l.dbgo[which / 2];
    CK(cudaMemcpyAsync(dst, src, need, cudaMemcpyDeviceToDevice, c->st));
    return SKIPPER_OK;
}

extern "C" size_t skipper_workspace_bytes(const skipper_layer *layers, int n, const skipper_config *cfg, int kept_max) {
    if (!layers || !cfg || n < 2) return 0;
    long long Nsum = 0, Nout_sum = 0;
    for (int i = 0; i < n - 1; ++i) {
        const skipper_layer &d = layers[i];
        long long N, No;
        if (d.kind == SKIPPER_LAYER_CONV3X3) {
            N = (long long)d.h * d.w * d.cout;
            No = d.pool == 2 ? N / 4 : N;
        } else {
            N = No = d.cout;
        }
        Nsum += N;
        Nout_sum += No;
    }
    const long long B = cfg->batch;
    const long long per_step = B * (Nsum * 4 + Nout_sum * 2);  // stored U fp32 + layer output bf16
    const long long per_ckpt = B * Nsum * 5;                   // checkpoint U fp32 + o u8
    if (cfg->mode == SKIPPER_MODE_FULL) return (size_t)(cfg->T * per_step);
    if (cfg->mode == SKIPPER_MODE_TBPTT) return (size_t)((cfg->C > 0 ? cfg->T / cfg->C : cfg->T) * per_step);
    const int C = cfg->C > 0 ? cfg->C : 1;
    const int rows = kept_max >= 0 ? kept_max : cfg->T / C;
    return (size_t)(C * per_ckpt + (long long)rows * per_step);
}

extern "C" skipper_status skipper_comm_unique_id(unsigned char id_out[128]) {
    std::string e;
    if (!sk::Comm::unique_id(id_out, &e)) return fail(nullptr, SKIPPER_ENCCL, "%s", e.c_str());
    return SKIPPER_OK;
}

static skipper_status comm_setup(skipper_ctx *c);

extern "C" skipper_status skipper_comm_init(skipper_ctx *c, const unsigned char id[128], int rank, int world) {
    CKS(check_ctx(c));
    if (world < 1 || rank < 0 || rank >= world) return fail(c, SKIPPER_EINVAL, "bad rank/world");
    // world == 1 also builds a (one-rank) communicator: the bucketed path then runs as an identity
    std::string e;
    if (!c->comm.init(id, rank, world, &e)) return fail(c, SKIPPER_ENCCL, "%s", e.c_str());
    return comm_setup(c);
}

extern "C" skipper_status skipper_comm_init_callback(skipper_ctx *c, skipper_allreduce_fn fn, void *user, int rank,
                                                     int world) {
    CKS(check_ctx(c));
    if (world < 1 || rank < 0 || rank >= world) return fail(c, SKIPPER_EINVAL, "bad rank/world");
    std::string e;
    if (!c->comm.init_callback(fn, user, rank, world, &e)) return fail(c, SKIPPER_EINVAL, "%s", e.c_str());
    return comm_setup(c);
}

// comm stream, events and the dW bucket plan (both communicator kinds)
static skipper_status comm_setup(skipper_ctx *c) {
    if (!c->st3 && cudaStreamCreateWithFlags(&c->st3, cudaStreamNonBlocking) != cudaSuccess)
        return fail(c, SKIPPER_ECUDA, "comm stream creation failed");
    if ((!c->ev_w && cudaEventCreateWithFlags(&c->ev_w, cudaEventDisableTiming) != cudaSuccess) ||
        (!c->ev_comm && cudaEventCreateWithFlags(&c->ev_comm, cudaEventDisableTiming) != cudaSuccess))
        return fail(c, SKIPPER_ECUDA, "comm event creation failed");
    std::vector<unsigned long long> wc(c->Ls);
    for (int i = 0; i < c->Ls; ++i) wc[i] = c->L[i].wcount;
    c->bucket_lo.assign(c->Ls, 0);
    static const unsigned long long kBucket = [] {
        const char *b = getenv("SKIPPER_BUCKET_MB");
        return (unsigned long long)(b ? std::max(1, atoi(b)) : 25) << 20;
    }();
    skipper_plan_buckets(wc.data(), c->Ls, kBucket, c->bucket_lo.data());
    return SKIPPER_OK;
}

// ------------------------------------------------------------------------------------ kernel-level API
// (include/skipper_kernels.h) - the same launchers skipper_step uses, for per-kernel parity tests.
static int kapi_run(const sk::GemmLaunch &g0, bool ok, void *stream, const char *what) {
    if (!ok) {
        g_last_error = std::string(what) + ": unsupported shape or tensor-map failure";
        return SKIPPER_EUNSUPPORTED;
    }
    sk::GemmLaunch g = g0;
    static unsigned long long *stats = nullptr;
    const char *se = getenv("SKIPPER_GEMM_STATS");
    if (se && atoi(se)) {  // diagnostics: per-role barrier wait cycles of this launch
        if (!stats) cudaMalloc(&stats, 8 * sizeof(unsigned long long));
        cudaMemsetAsync(stats, 0, 8 * sizeof(unsigned long long), static_cast<cudaStream_t>(stream));
        g.d.stats = stats;
    }
    cudaError_t e = sk::gemm_run(g, static_cast<cudaStream_t>(stream), sk::device_num_sms());
    if (g.d.stats && e == cudaSuccess) {
        unsigned long long h[8];
        cudaMemcpyAsync(h, stats, sizeof h, cudaMemcpyDeviceToHost, static_cast<cudaStream_t>(stream));
        cudaStreamSynchronize(static_cast<cudaStream_t>(stream));
        const double cta = (double)h[3];
        fprintf(stderr, "[gemm-stats %s] bn=%d mn=%d cs=%d tiles=%d kb=%d: producer<-empty %.2f  mma<-tmem %.2f  mma<-data %.2f  epi<-acc %.2f (fractions of CTA cycles)\n",
                what, g.bn, g.mn_major, g.cs, g.d.m_tiles * g.d.n_tiles * g.d.taps * g.d.splits, g.d.kb_per_split,
                h[0] / cta, h[1] / cta, h[4] / cta, h[2] / (4 * cta));
    }
    if (e != cudaSuccess) {
        g_last_error = std::string(what) + ": " + cudaGetErrorString(e);
        return SKIPPER_ECUDA;
    }
    return SKIPPER_OK;
}

extern "C" int skipper_k_fc_fwd(const unsigned short *A, const unsigned short *B, float *C, int M, int N, int K,
                                void *stream) {
    sk::GemmLaunch g;
    const bool ok = sk::plan_fc(&g, A, B, C, M, N, K);
    return kapi_run(g, ok, stream, "fc_fwd");
}

extern "C" int skipper_k_fc_wgrad(const unsigned short *D, const unsigned short *X, float *dW, int M, int N, int K,
                                  int accumulate, void *stream) {
    if (!accumulate && cudaMemsetAsync(dW, 0, (size_t)N * K * 4, static_cast<cudaStream_t>(stream)) != cudaSuccess)
        return SKIPPER_ECUDA;
    sk::GemmLaunch g;
    const bool ok = sk::plan_fc_wgrad(&g, D, X, dW, M, N, K, sk::device_num_sms());
    return kapi_run(g, ok, stream, "fc_wgrad");
}

extern "C" int skipper_k_conv_fwd(const unsigned short *X, const unsigned short *Wk, float *Y, int nb, int h, int w,
                                  int cin, int cout, void *stream) {
    sk::GemmLaunch g;
    const bool ok = sk::plan_conv(&g, X, Wk, Y, nb, h, w, cin, cout, +1);
    return kapi_run(g, ok, stream, "conv_fwd");
}

extern "C" int skipper_k_conv_lif(const unsigned short *X, const unsigned short *Wk, float *U_state,
                                  unsigned char *o_state, unsigned short *P, float *U_out, int R, int nb, int h, int w,
                                  int cin, int cout, int pool, float lam, float theta, void *stream) {
    if (!sk::conv_lif_supported(nb, h, w, cin, cout, pool)) {
        g_last_error = "conv_lif: unsupported shape";
        return SKIPPER_EUNSUPPORTED;
    }
    sk::ConvLifArgs a{};
    a.B = nb;
    a.H = h;
    a.W = w;
    a.Cin = cin;
    a.Cout = cout;
    a.pool = pool;
    a.R = R;
    a.U_state = U_state;
    a.o_state = o_state;
    a.U_out = U_out;
    a.Po_out = P;
    a.lam = lam;
    a.theta = theta;
    cudaError_t e = sk::launch_conv_lif(X, R, Wk, a, static_cast<cudaStream_t>(stream), sk::device_num_sms());
    if (e != cudaSuccess) {
        g_last_error = std::string("conv_lif: ") + cudaGetErrorString(e);
        return SKIPPER_ECUDA;
    }
    return SKIPPER_OK;
}

extern "C" int skipper_k_conv_dgrad(const unsigned short *D, const unsigned short *Wt, float *G, int nb, int h, int w,
                                    int cin, int cout, void *stream) {
    sk::GemmLaunch g;
    const bool ok = sk::plan_conv(&g, D, Wt, G, nb, h, w, cout, cin, -1);
    return kapi_run(g, ok, stream, "conv_dgrad");
}

extern "C" int skipper_k_conv_wgrad(const unsigned short *D, const unsigned short *X, float *dW, int nb, int h, int w,
                                    int cin, int cout, int accumulate, void *stream) {
    if (!accumulate && cudaMemsetAsync(dW, 0, (size_t)cout * 9 * cin * 4, static_cast<cudaStream_t>(stream)) != cudaSuccess)
        return SKIPPER_ECUDA;
    sk::GemmLaunch g;
    const bool ok = sk::plan_conv_wgrad(&g, D, X, dW, nb, h, w, cin, cout, sk::device_num_sms());
    return kapi_run(g, ok, stream, "conv_wgrad");
}

extern "C" int skipper_k_narrow_wgrad(const unsigned short *D, const unsigned short *X, float *dW, int nb, int h, int w,
                                      int cin, int cout, int stride, int accumulate, void *stream) {
    if (!sk::narrow_wgrad_supported(cin, cout, stride, h, w)) {
        g_last_error = "narrow_wgrad: unsupported shape";
        return SKIPPER_EUNSUPPORTED;
    }
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    const size_t cnt = (size_t)cout * 9 * cin;
    if (!accumulate && cudaMemsetAsync(dW, 0, cnt * 4, st) != cudaSuccess) return SKIPPER_ECUDA;
    // the kernel writes one dW slice per CTA; sum them in slice order (as the engine does)
    const int ns = sk::narrow_wgrad_slices(cin, cout, stride, h, w, sk::device_num_sms());
    float *sl = nullptr;
    if (ns < 1 || cudaMallocAsync(reinterpret_cast<void **>(&sl), (size_t)ns * cnt * 4, st) != cudaSuccess ||
        cudaMemsetAsync(sl, 0, (size_t)ns * cnt * 4, st) != cudaSuccess) {
        g_last_error = "narrow_wgrad: slice allocation failed";
        return SKIPPER_ECUDA;
    }
    const bool ok = sk::launch_narrow_wgrad(reinterpret_cast<const uint16_t *>(X), reinterpret_cast<const uint16_t *>(D), sl,
                                            nb, h, w, cin, cout, stride, st, sk::device_num_sms()) == cudaSuccess &&
                    sk::launch_reduce_slices(sl, ns, dW, cnt, st) == cudaSuccess;
    cudaFreeAsync(sl, st);
    if (!ok) {
        g_last_error = "narrow_wgrad: launch failed";
        return SKIPPER_ECUDA;
    }
    return SKIPPER_OK;
}

extern "C" int skipper_k_narrow_dgrad(const unsigned short *D, const unsigned short *Wt, float *G, int nb, int h, int w,
                                      int cin, int cout, int stride, void *stream) {
    if (!sk::narrow_dgrad_supported(cin, cout, h, w, stride)) {
        g_last_error = "narrow_dgrad: unsupported shape";
        return SKIPPER_EUNSUPPORTED;
    }
    if (sk::launch_narrow_dgrad(reinterpret_cast<const uint16_t *>(D), reinterpret_cast<const uint16_t *>(Wt), G, nb, h, w,
                                cin, cout, stride, static_cast<cudaStream_t>(stream), sk::device_num_sms()) != cudaSuccess) {
        g_last_error = "narrow_dgrad: launch failed";
        return SKIPPER_ECUDA;
    }
    return SKIPPER_OK;
}

extern "C" int skipper_k_conv_s(const unsigned short *X, const unsigned short *Wk, float *Y, int nb, int h, int w,
                                int cin, int cout, int sign, int stride, void *stream) {
    sk::GemmLaunch g;
    const bool ok = sk::plan_conv_s(&g, X, Wk, Y, nb, h, w, cin, cout, sign, stride);
    return kapi_run(g, ok, stream, "conv_s");
}

extern "C" int skipper_k_conv_narrow(const unsigned short *X, const unsigned short *Wk, float *Y, int nb, int h, int w,
                                     int cin, int cout, int sign, int stride, void *stream) {
    if (!sk::conv_narrow_supported(cin, cout, stride, sign)) {
        g_last_error = "conv_narrow: unsupported shape";
        return SKIPPER_EUNSUPPORTED;
    }
    sk::NarrowConvArgs a{};
    a.X = X;
    a.Wk = Wk;
    a.Y = Y;
    a.nb = nb;
    a.H = h;
    a.W = w;
    a.Hin = h * stride;
    a.Win = w * stride;
    a.Cin = cin;
    a.Cout = cout;
    a.stride = stride;
    a.sign = sign;
    const cudaError_t e = sk::launch_conv_narrow(a, static_cast<cudaStream_t>(stream), sk::device_num_sms());
    if (e != cudaSuccess) {
        g_last_error = std::string("conv_narrow: ") + cudaGetErrorString(e);
        return SKIPPER_ECUDA;
    }
    return SKIPPER_OK;
}

extern "C" int skipper_k_num_sms(void) { return sk::device_num_sms(); }

// ------------------------------------------------------------------------------------ profiling API
extern "C" skipper_status skipper_profile(skipper_ctx *c, int enable) {
    CKS(check_ctx(c));
    prof_resolve(c);
    c->prof_on = enable != 0;
    c->prof_log.clear();
    for (int k = 0; k < 16; ++k) {
        c->prof_n[k] = 0;
        c->prof_ms[k] = c->prof_bytes[k] = c->prof_flops[k] = 0;
    }
    return SKIPPER_OK;
}

extern "C" skipper_status skipper_profile_read(skipper_ctx *c, int cls, long long *launches, double *ms, double *bytes,
                                               double *flops) {
    CKS(check_ctx(c));
    if (cls < 0 || cls >= K_NCLASS) return fail(c, SKIPPER_EINVAL, "kernel class %d out of range", cls);
    prof_resolve(c);
    if (launches) *launches = c->prof_n[cls];
    if (ms) *ms = c->prof_ms[cls];
    if (bytes) *bytes = c->prof_bytes[cls];
    if (flops) *flops = c->prof_flops[cls];
    return SKIPPER_OK;
}

// The profiled scopes since skipper_profile() in launch order: class, kernels launched in the scope,
// algorithmic bytes / FLOPs, device ms (CUDA events).  Fills up to cap entries; returns the total count.
extern "C" long long skipper_profile_records(skipper_ctx *c, int *cls, long long *nk, double *bytes, double *flops,
                                            float *ms, long long cap) {
    if (!c) return -1;
    prof_resolve(c);
    const long long n = (long long)c->prof_log.size();
    for (long long i = 0; i < n && i < cap; ++i) {
        const auto &r = c->prof_log[i];
        if (cls) cls[i] = r.cls;
        if (nk) nk[i] = r.nk;
        if (bytes) bytes[i] = r.bytes;
        if (flops) flops[i] = r.flops;
        if (ms) ms[i] = r.ms;
    }
    return n;
}

extern "C" const char *skipper_profile_class_name(int cls) {
    if (cls < 0 || cls >= K_NCLASS) return nullptr;
    return k_class_names[cls];
}

extern "C" int skipper_profile_num_classes(void) { return K_NCLASS; }

extern "C" long long skipper_launch_count(const skipper_ctx *c) { return c ? c->launches : 0; }
