/*
 * skipper.h - C ABI of the B200 (sm_100a) Skipper SNN training hot path.
 *
 * Paper: Singh et al., "Skipper: Enabling efficient SNN training through
 * activation-checkpointing and time-skipping", MICRO 2022.  Citations P:<n>
 * are lines of the paper text; SURVEY.md §8 is the scope contract.
 *
 * What one training iteration computes (skipper_step):
 *   FIRST forward pass over t = 0..T-1 (Fig. 5/6 Step 1):
 *     LIF dynamics, Eq.1:  U_t = lam*U_{t-1} + W o^{l-1}_t - theta*o_{t-1},
 *     o_t = [U_t > theta]; the state (U, o) of every spiking layer is stored only at
 *     the segment starts t = cS (the checkpoints); SAM spike sums s_t, Eq.4.
 *   readout + loss at t = T-1 (readout reading 5 of SURVEY.md §8(c)).
 *   SST_c, Eq.5, keep t iff s_t > SST_c [mode SKIP].
 *   for c = C-1..0: RECOMPUTE the kept steps of segment c from its checkpoint
 *     (P:742-748), then BACKWARD through them with the surrogate
 *     gradient, Eq.2, carrying dL/dU of the segment start to c-1
 *     (P:750-753); segment memory is released.
 *   data-parallel gradient allreduce and Adam.
 *
 * Conventions
 *   - Pointers named *_dev are CUDA device pointers, *_host are host pointers.
 *   - Every call is stream-ordered on the stream given to skipper_create, except
 *     the calls documented as synchronising (they say "host sync").
 *   - Layouts are row-major, NHWC for images.  Input spikes x are uint8 {0,1}
 *     of shape [T][B][H][W][C] (conv first layer) or [T][B][D] (fc first layer),
 *     B = cfg.batch (the per-rank batch).  Labels are int32 [B].
 *   - Weights are float32, per layer:  fc [cout][cin];  conv [cout][3][3][cin];
 *     readout [classes][cin].  fc layers read the previous conv output flattened
 *     in (h, w, c) order.
 *   - Ownership: the caller owns x, labels and any output buffer and keeps them
 *     alive until the stream reaches the call.  The context owns all state and
 *     workspace and allocates device memory through the allocator given at
 *     creation (NULL -> cudaMallocAsync on the context stream).
 *   - Errors: every call returns a skipper_status; skipper_last_error() gives the
 *     message.  A CUDA or NCCL error poisons the context (later calls return
 *     SKIPPER_EFAILED).  Argument or call-order errors leave the weights untouched.
 *   - A context is not thread-safe; use one per rank / per thread.
 */
#ifndef SKIPPER_H
#define SKIPPER_H

#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct skipper_ctx skipper_ctx;

typedef enum {
    SKIPPER_OK = 0,
    SKIPPER_EINVAL = 1,       /* invalid argument / configuration                  */
    SKIPPER_ENOMEM = 2,       /* allocator returned NULL                            */
    SKIPPER_ECUDA = 3,        /* CUDA error (context poisoned)                      */
    SKIPPER_ENCCL = 4,        /* NCCL error (context poisoned)                      */
    SKIPPER_EORDER = 5,       /* segment calls out of the order Fig. 5/6 require    */
    SKIPPER_EFAILED = 6,      /* context previously poisoned                        */
    SKIPPER_EUNSUPPORTED = 7  /* layer geometry this build has no kernel for        */
} skipper_status;

/* TBPTT (Sec. III-C): C truncation windows of t' = T/C steps;
 * each window integrates its own readout (z_w = W^L sum_{t in w} a_t / t'), adds its cross-entropy to the
 * loss and back-propagates through the window only (delta is zero after the window's last step); the
 * neuron state carries on; weight gradients are summed over windows.  Segment API order:
 * forward_segment(w, FIRST, x, labels) then backward_segment(w) for w = 0..C-1, then optimizer_step. */
typedef enum { SKIPPER_MODE_FULL = 0, SKIPPER_MODE_CKPT = 1, SKIPPER_MODE_SKIP = 2, SKIPPER_MODE_TBPTT = 3 } skipper_mode;
typedef enum { SKIPPER_PASS_FIRST = 0, SKIPPER_PASS_RECOMPUTE = 1, SKIPPER_PASS_RECORD = 2 } skipper_pass;
typedef enum { SKIPPER_LAYER_FC = 0, SKIPPER_LAYER_CONV3X3 = 1, SKIPPER_LAYER_READOUT = 2 } skipper_layer_kind;
typedef enum { SKIPPER_SURR_TRIANGLE = 0, SKIPPER_SURR_FAST_SIGMOID = 1 } skipper_surrogate;
/* Spike Activity Monitor metric the skip policy thresholds (Eq.5 takes the percentile of it):
 * SPIKES   s_t = sum over the input and every spiking layer of the spikes at t (Eq.4);
 * WEIGHTED s_t = sum_l count_l,t / N_l, N_l = neurons per sample of layer l (l = 0: the input), in
 *          float64 in layer order - "the sum of spike counts weighted by the neuron count in each
 *          layer" (reading 22).
 * L2TRACE  s_t = sqrt(sum over every spiking neuron of U_t^2), the l2 norm of the membrane trace at t (the
 *          other variant P:1049-1061 names; reading 25), squares exact in float64, summed in
 *          float64 (allreduced under DP); the mask then depends only on the order of the s_t. */
typedef enum { SKIPPER_SAM_SPIKES = 0, SKIPPER_SAM_WEIGHTED = 1, SKIPPER_SAM_L2TRACE = 2 } skipper_sam;

/* One layer.  conv3x3: zero pad 1, stride 1 or 2; h x w = the OUTPUT (neuron) size, the
 * input is (stride*h) x (stride*w); optional 2x2 average pooling of the output spikes
 * (pool = 2).  fc: h = w = 1.  The last layer must be the (non-spiking) readout;
 * lambda/theta are ignored for it, and pool = 1 on the readout means it integrates the
 * global average pool of the last conv layer's spikes (reading 23; then cin = that
 * layer's cout).
 * residual_from (ResNet SNN, Table I "ResNet20", reading 8): -1, or the index
 * r = (this layer) - 2 of a spiking conv layer whose output spikes are added into this
 * layer's current through the option-A shortcut: subsample by h_r / h (1 or 2) and
 * zero-pad the channels (cout - cout_r) / 2 on each side.  Unpooled layers only. */
typedef struct {
    int kind;        /* skipper_layer_kind */
    int cin, cout;
    int h, w;
    int pool;        /* 0 or 2 (conv); 0 or 1 = GAP (readout) */
    float lambda;    /* leak, Eq.1 (lambda < 1; 1 = integrate-and-fire) */
    float theta;     /* firing threshold, Eq.1 */
    int stride;      /* conv: 1 or 2 (0 is read as 1) */
    int residual_from;  /* -1 or layer index - 2 (see above) */
} skipper_layer;

typedef struct {
    int T;                 /* timesteps */
    int C;                 /* checkpoints = segments; T % C == 0, C < T/L_n */
    double p;              /* SST percentile in [0, 100); 0 => no skipping (Eq.5) */
    int mode;              /* skipper_mode (FULL ignores C and p) */
    int batch;             /* per-rank batch B */
    int global_batch;      /* loss normaliser (sum over ranks of batch); 0 => batch */
    int surrogate;         /* skipper_surrogate */
    float surr_gamma;      /* triangle: peak; fast sigmoid: slope */
    float lr, beta1, beta2, eps;   /* Adam */
    int debug_record;      /* 1: keep per-step states for skipper_debug_copy (tests) */
    int sam;               /* skipper_sam (0 = Eq.4 spike sum) */
    int group;             /* CKPT / SKIP backward groups: segments recomputed (one at a time) into one arena and
                              back-propagated as one layer-major pass over their concatenated rows.  0 or 1 =
                              the paper's schedule (one segment at a time); G > 1 trades a G-times
                              larger segment arena (still O(T/C), Eq.6) for fewer, longer backward launches.
                              The gradients are those of the per-segment schedule (the reverse scan carries
                              delta across segment borders exactly as the per-segment carry does). */
} skipper_config;

/* Device-memory allocator used for every context allocation. */
typedef struct {
    void *(*alloc)(size_t bytes, void *stream, void *user);
    void (*free)(void *ptr, size_t bytes, void *stream, void *user);
    void *user;
} skipper_allocator;

/* Create a context: validates the network and configuration (EINVAL with a
 * message on failure; a p above the Eq.7 bound is accepted and
 * reported by skipper_last_error as a warning), allocates weights, optimizer
 * moments, checkpoint store and persistent buffers.  Weights start at zero:
 * call skipper_set_weights for every layer.  cuda_stream may be NULL (legacy
 * default stream).  On failure *out is NULL and the message is available from
 * skipper_last_error(NULL). */
skipper_status skipper_create(const skipper_layer *layers, int n_layers, const skipper_config *cfg,
                              const skipper_allocator *alloc, void *cuda_stream, skipper_ctx **out);
void skipper_destroy(skipper_ctx *ctx);
const char *skipper_last_error(const skipper_ctx *ctx);   /* ctx may be NULL */

/* Weights, float32 on the device, layout per the conventions above.  set copies
 * into the fp32 master and refreshes the bf16 shadows used by the tensor cores;
 * it resets nothing else.  get_grads returns dL/dW of the last completed
 * backward (summed over ranks after skipper_optimizer_step / skipper_step). */
skipper_status skipper_set_weights(skipper_ctx *ctx, int layer, const float *w_dev);
skipper_status skipper_get_weights(skipper_ctx *ctx, int layer, float *w_dev);
skipper_status skipper_get_grads(skipper_ctx *ctx, int layer, float *dw_dev);
size_t skipper_weight_count(const skipper_ctx *ctx, int layer);

/* ---- segment-level calls (the pieces skipper_step composes) ----------------
 * Order (EORDER otherwise):
 *   CKPT/SKIP: forward_segment(c, FIRST) for c = 0..C-1 (the call for c = C-1
 *              takes labels_dev, computes the loss and dL/dz, allreduces s over
 *              ranks and fixes the keep mask - one host sync);
 *              then for c = C-1..0: forward_segment(c, RECOMPUTE), backward_segment(c);
 *              then optimizer_step.
 *   FULL:      forward_segment(0, RECORD) (all T steps stored, takes labels_dev),
 *              backward_segment(0), optimizer_step.
 * x_dev is the whole input [T][B][...] (uint8) and must be the same pointer
 * contents for every call of one iteration. */
skipper_status skipper_forward_segment(skipper_ctx *ctx, int seg, int pass,
                                       const unsigned char *x_dev, const int *labels_dev);
skipper_status skipper_backward_segment(skipper_ctx *ctx, int seg);
/* Join the dW allreduce (issued in buckets during backward_segment(0) when skipper_comm_init was
 * called) and apply Adam. */
skipper_status skipper_optimizer_step(skipper_ctx *ctx);

/* One full training iteration on device-resident inputs.  loss_host may be NULL
 * (then the only host sync of the step is the one that fixes the keep mask). */
skipper_status skipper_step(skipper_ctx *ctx, const unsigned char *x_dev, const int *labels_dev,
                            float *loss_host);
/* Same, end to end from host memory: copies x [T][B][...] and labels to the
 * device inside the call (pinned host memory gives asynchronous copies), runs
 * the step and copies the loss back (host sync). */
skipper_status skipper_step_host(skipper_ctx *ctx, const unsigned char *x_host, const int *labels_host,
                                 float *loss_host);

/* ---- on-device input encoding ----------
 * Poisson rate coding o0_t[b][d] = [u < x[b][d] * rates[t]] with u drawn from Philox4x32-10:
 * element e of the row-major [T][B][D] output uses word e%4 of Philox(counter = (e/4 lo, e/4 hi, 0, 0),
 * key = (seed lo, seed hi)), u = (word >> 8) * 2^-24; x * rates[t] is one fp32 product (reading 18;
 * oracle/encoder.py draws the identical numbers).  x_dev: float32 [B][D] intensities in [0, 1] (D = the
 * input elements per sample), rates_dev: float32 [T]; out_dev: uint8 [T][B][D].  All device pointers. */
skipper_status skipper_encode_poisson(const float *x_dev, const float *rates_dev, unsigned long long seed, int T,
                                      int B, long long D, unsigned char *out_dev, void *stream);
/* One training iteration from intensities: encodes the spikes into a context-owned buffer on the context
 * stream, then skipper_step.  skipper_step_host_encoded: the same from host buffers (H2D of x, rates and
 * labels inside the call, then the loss D2H) - the end-to-end user call. */
skipper_status skipper_step_encoded(skipper_ctx *ctx, const float *x_dev, const float *rates_dev, unsigned long long seed,
                                    const int *labels_dev, float *loss_host);
skipper_status skipper_step_host_encoded(skipper_ctx *ctx, const float *x_host, const float *rates_host,
                                         unsigned long long seed, const int *labels_host, float *loss_host);

/* ---- data parallelism (batch-sharded) ----------
 * comm_unique_id: rank 0 creates the NCCL id; the caller broadcasts it.  comm_init: every rank joins
 * the library-owned communicator (world == 1 builds a one-rank communicator: the same schedule runs and
 * the collectives are identities).  With a communicator, the per-layer spike counts are allreduced
 * (int64) before Eq.5 so every rank computes the same keep mask, and dW is allreduced (fp32 sum) in
 * layer buckets of SKIPPER_BUCKET_MB (default 25) on a dedicated stream as soon as segment 0's weight
 * gradients of the bucket's layers have run, overlapping the rest of the backward.  ENCCL on failure
 * (the context is then poisoned). */
skipper_status skipper_comm_unique_id(unsigned char id_out[128]);
skipper_status skipper_comm_init(skipper_ctx *ctx, const unsigned char id[128], int rank, int world);
/* The same data-parallel schedule with the collectives delegated to a host callback instead of NCCL:
 * fn(buf_dev, count, dtype (0 f32, 1 f64, 2 int64), stream, user) must sum `count` elements at buf_dev
 * over all ranks in place, ordered after the work already issued to `stream` (a cudaStream_t) and complete
 * when it returns; it returns 0 on success (else the call fails with ENCCL).  For process groups NCCL cannot
 * serve - several ranks on one GPU (tests: torch.distributed gloo), or a host-side transport. */
typedef int (*skipper_allreduce_fn)(void *buf_dev, size_t count, int dtype, void *stream, void *user);
skipper_status skipper_comm_init_callback(skipper_ctx *ctx, skipper_allreduce_fn fn, void *user, int rank, int world);
/* The bucket plan (host only): walking spiking layers n_spiking-1 .. 1, closes[i] = 1 where a bucket of
 * >= bucket_bytes of fp32 gradients ends (layer 1 always ends the last one; layer 0 and the readout go
 * after segment 0).  Returns the number of buckets, or -1 for null pointers or n_spiking < 1. */
int skipper_plan_buckets(const unsigned long long *wcount, int n_spiking, unsigned long long bucket_bytes,
                         int *closes);

/* ---- introspection (host sync) ----------------------------------------------- */
skipper_status skipper_get_loss(skipper_ctx *ctx, float *loss_host);
skipper_status skipper_get_spike_sums(skipper_ctx *ctx, long long *s_host);      /* [T], global */
/* per-layer spike counts of the last first pass, [L_n + 1][T] (row 0 = input spikes), global batch */
skipper_status skipper_get_layer_spike_counts(skipper_ctx *ctx, long long *counts_host);
/* the SAM values the keep mask was computed from (cfg.sam metric), [T] float64 */
skipper_status skipper_get_sam(skipper_ctx *ctx, double *sam_host);
skipper_status skipper_get_keep_mask(skipper_ctx *ctx, unsigned char *keep_host); /* [T] */
skipper_status skipper_get_sst(skipper_ctx *ctx, double *sst_host);               /* [C]; NaN if p == 0 */
skipper_status skipper_mem_stats(skipper_ctx *ctx, size_t *current_bytes, size_t *peak_bytes);
skipper_status skipper_reset_peak(skipper_ctx *ctx);

/* Debug copies (require cfg.debug_record = 1), device to device:
 *   which 0: first-pass U   float32 [T][B*N_l]
 *   which 1: first-pass o   uint8   [T][B*N_l]
 *   which 2: recomputed U   float32 [T][B*N_l]  (rows of kept t; others 0)
 *   which 3: recomputed o   uint8   [T][B*N_l]
 * N_l is the un-pooled neuron count of spiking layer `layer` (0-based). */
skipper_status skipper_debug_copy(skipper_ctx *ctx, int which, int layer, void *dst_dev, size_t bytes);

/* ---- profiling (bench / roofline) --------------------------------------------
 * enable != 0: every kernel launch of the context is bracketed by CUDA events on
 * the context stream and attributed to a kernel class, with its algorithmic HBM
 * bytes and FLOPs.  Counters reset on every call.
 * profile_read synchronises the stream (host sync) and returns the totals of one
 * class since the last reset.  Classes are numbered 0..skipper_profile_num_classes()-1. */
skipper_status skipper_profile(skipper_ctx *ctx, int enable);
skipper_status skipper_profile_read(skipper_ctx *ctx, int cls, long long *launches, double *ms, double *bytes,
                                    double *flops);
const char *skipper_profile_class_name(int cls);
int skipper_profile_num_classes(void);
/* The profiled scopes since the last skipper_profile() call, in launch order: kernel class, number of
 * kernels the scope launched, algorithmic bytes and FLOPs, device ms.  Host arrays of `cap` entries (any
 * may be NULL); synchronises the stream; returns the total number of scopes (-1 on a null context).  Used
 * to attribute an ncu launch list to kernel classes (tools/ncu_classes.py). */
long long skipper_profile_records(skipper_ctx *ctx, int *cls, long long *n_kernels, double *bytes, double *flops,
                                  float *ms, long long cap);
/* Kernel launches issued by this context since creation (always counted). */
long long skipper_launch_count(const skipper_ctx *ctx);

/* Pure host functions (no GPU needed). */
/* Eq.5 for one segment: p-th percentile of n int64 values, numpy 'linear' method. */
double skipper_sst_host(const long long *s, int n, double p);
/* Stored neuron-state bytes at the peak for a mode (the Eq.3 / Eq.6 model with
 * this build's storage: fp32 U + bf16 output per stored step, fp32 U + u8 o per
 * checkpoint); kept_max < 0 means T/C. */
size_t skipper_workspace_bytes(const skipper_layer *layers, int n_layers, const skipper_config *cfg,
                               int kept_max);
const char *skipper_status_string(int status);
const char *skipper_build_info(void);

#ifdef __cplusplus
}
#endif
#endif /* SKIPPER_H */
