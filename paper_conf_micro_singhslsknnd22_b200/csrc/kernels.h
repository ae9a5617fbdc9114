// kernels.h - launchers for the non-GEMM kernels of the hot path (all sm_100a CUDA cores).
#pragma once
#include <cstddef>
#include <cstdint>
#include <cuda_runtime.h>

namespace sk {

enum { SURR_TRIANGLE = 0, SURR_FAST_SIGMOID = 1 };

// K1: forward LIF temporal scan over the rows (timesteps) of one segment, Eq.1.
// Neuron layout NHWC per row: row r holds B*H*W*C neurons (fc: H = W = 1).
struct ScanFwdArgs {
    const float *I;        // currents [R][B*N]
    int nsplit;            // I is the fixed-order sum of nsplit partial slices (deterministic split-K)
    long long split_stride;  // floats between partial slices
    int R;                 // rows in the segment buffer
    int restore;           // RECOMPUTE: row 0 is the checkpoint (U_state/o_state), rows 1.. recomputed
    float *U_state;        // FIRST/RECORD: running U [B*N] (in/out); RECOMPUTE: checkpoint U (in)
    uint8_t *o_state;      // same for spikes
    float *U_out;          // [R][B*N] stored membranes (RECOMPUTE/RECORD) or null
    uint16_t *Po_out;      // [R][B*Nout] bf16 layer output (pooled if pool) - next GEMM operand
    float *ckU;            // FIRST: checkpoint slot written after row 0, else null
    uint8_t *cko;
    int ck_every;          // >0: rows r % ck_every == 0 write checkpoint slot r / ck_every (whole-T scans)
    unsigned *s_part;      // SAM partials [T][32] or null (FIRST/RECORD only)
    double *u2_part;       // l2-trace SAM (reading 25): sum of U^2 per row into [T][32] fp64 partials, or null
    const int *row_t;      // absolute t of each row (device) or null -> t0 + r
    int t0;
    float *cnt;            // readout accumulation [B*Nout] or null (last spiking layer)
    float *dbg_U;          // debug [T][B*N] or null
    uint8_t *dbg_o;
    int B, H, W, C, pool;
    float lam, theta;
    // ResNet residual (reading 8): I += S(a^r), the option-A shortcut of the bf16 output rows of source
    // layer r, [R][B][res_H][res_W][res_C] (row r of the segment reads row r); unpooled layers only
    const uint16_t *res;
    int res_H, res_W, res_C, res_stride, res_lo;
};
cudaError_t launch_lif_fwd(const ScanFwdArgs &a, cudaStream_t s);

// K4: reverse surrogate-gradient scan, Eq.2: delta_t = sigma'(U_t) g_t + lam delta_{next}.
struct ScanBwdArgs {
    const float *g;        // gradient wrt the layer's output spikes
    int nsplit;            // g = sum of nsplit partial slices, split_stride floats apart
    long long split_stride;
    int g_pooled;          // g is at pooled resolution (x 0.25 spread, pool2^T)
    int g_broadcast;       // g is [B*Nout] for every row (readout gradient, same at each t)
    const float *U;        // [R][B*N]
    float *carry;          // [B*N] delta at the first row of the next segment (in) / of this one (out)
    uint16_t *delta;       // [R][B*N] bf16 (dgrad / wgrad operand) or null
    int R;
    int B, H, W, C, pool;
    float lam, theta;
    int surr;
    float gamma;
    // ResNet residual (reading 8): this layer is the shortcut source of a later layer whose bf16 delta
    // rows res_delta [R][B][H/res_stride][W/res_stride][res_C] add S^T(delta) to g (unpooled layers only)
    const uint16_t *res_delta;
    int res_C, res_stride, res_lo;
};
cudaError_t launch_lif_bwd(const ScanBwdArgs &a, cudaStream_t s);

// Layer-0 operand rows of one segment straight from the uint8 input x [T][B][...]:
// kind 0: bf16 copy of x[t] (D = elements per sample); kind 1: 3x3/pad-1 im2col of an
// H x W x C0 image zero-padded to K0 columns.  rows: device list of t (or null -> t0 + r).
// s_part != null adds the SAM term l = 0 (Eq.4).
// kind 1 with stride 2: H x W are the OUTPUT pixels, the image is (2H) x (2W); SAM counts every input pixel.
cudaError_t launch_stage_rows(const uint8_t *x, uint16_t *dst, const int *rows, int t0, int R, int B, int H, int W,
                              int C0, int kind, int K0, long long D, unsigned *s_part, cudaStream_t s, int stride = 1);

// Narrow / strided conv layers (ResNet SNN): explicit 3x3 im2col of bf16 NHWC rows,
// cols[(n, y, x)][(dy*3+dx)*Cin + ci] = X[n][s*y+dy-1][s*x+dx-1][ci] (zero outside), Cin % 8 == 0.
// Narrow-channel (cin 16 / 32) 3x3 conv weight gradient without a column buffer (narrow_wgrad.cu):
// dW[cout][9][cin] += sum over the nb*H*W output pixels of D[.][cout] X_shift[.][cin]; X is the layer
// input [nb][H*stride][W*stride][cin], D [nb][H][W][cout], both bf16.
bool narrow_wgrad_supported(int cin, int cout, int stride, int H, int W);
// dW slices the narrow weight gradient writes: CTA b adds its partial into dW + b * |dW| (deterministic; sum
// the slices with launch_reduce_slices)
int narrow_wgrad_slices(int cin, int cout, int stride, int H, int W, int num_sms);
// dst[i] += sum_{s < nslices} slices[s * count + i] in slice order, then slices[s * count + i] = 0
// zero = 0: the slices are left as they are (the engine clears them at the start of the next step, off the
// critical path)
cudaError_t launch_reduce_slices(float *slices, int nslices, float *dst, size_t count, cudaStream_t s, int zero = 1);
cudaError_t launch_narrow_wgrad(const uint16_t *X, const uint16_t *D, float *dW, int nb, int H, int W, int cin,
                                int cout, int stride, cudaStream_t s, int num_sms);
// dgrad of a narrow 3x3 conv, stride 1 or 2 (narrow_wgrad.cu): G [nb][s*H][s*W][cin] fp32 from the layer's
// delta D [nb][H][W][cout] and the transposed weights Wt [cin][9][cout]; cin 16 / 32, cout 16 / 32 (64 for
// cin 32 at stride 2)
bool narrow_dgrad_supported(int cin, int cout, int H, int W, int stride);
cudaError_t launch_narrow_dgrad(const uint16_t *D, const uint16_t *Wt, float *G, int nb, int H, int W, int cin, int cout,
                                int stride, cudaStream_t s, int num_sms);
cudaError_t launch_im2col_bf16(const uint16_t *X, uint16_t *cols, long long nb, int Hin, int Win, int Cin, int H,
                               int W, int stride, cudaStream_t s);
// Adjoint: G[n][yi][xi][ci] = sum_{dy,dx: s | (yi+1-dy), s | (xi+1-dx)} dcols[(n, y, x)][ci*9 + dy*3+dx]
// (column order (ci, tap): the dgrad GEMM's B operand is the transposed shadow [cin][9][cout]).
cudaError_t launch_col2im_f32(const float *dcols, float *G, long long nb, int Hin, int Win, int Cin, int H, int W,
                              int stride, cudaStream_t s);
// Global average pool of the readout input (reading 23): out[b][c] = sum_p in[b][p][c] / P, and its adjoint.
cudaError_t launch_gap_reduce(const float *in, float *out, int B, int P, int C, cudaStream_t s);
cudaError_t launch_gap_expand(const float *g, float *out, int B, int P, int C, cudaStream_t s);
cudaError_t launch_cast_pad_bf16(const float *src, uint16_t *dst, int rows, int cols, int ld, cudaStream_t s);
cudaError_t launch_unpad_f32(const float *src, float *dst, int rows, int cols, int ld, cudaStream_t s);
cudaError_t launch_sam_finalize(const unsigned *s_part, long long *s, int T, cudaStream_t st);
// Poisson rate encoder (NEXT-3): out[t][b][d] = [u < x[b][d] * rates[t]], u from Philox4x32-10
cudaError_t launch_poisson_encode(const float *x, const float *rates, unsigned long long seed, int T, int B, long long D,
                                  uint8_t *out, cudaStream_t s);
// u2[t] = sum of the 32 fp64 partials of row t, in slot order
cudaError_t launch_sum32_f64(const double *part, double *out, int T, cudaStream_t st);

// Fused first layer for narrow inputs (layer0.cu): im2col in smem + tcgen05 + LIF + pool + SAM.
struct L0FwdArgs {
    const uint8_t *x;      // input spikes [T][B][H][W][C0]
    int T, B, H, W, C0;
    const int *row_t;      // absolute t per row (device) or null -> t0 + r
    int t0, R, restore;    // restore: row 0 is the checkpoint (U_state/o_state), no MMA for it
    const uint16_t *wbp;   // bf16 weights [N][32] (k = (dy*3+dx)*C0 + ci, zero padded)
    int N, pool;
    float lam, theta;
    float *U_state;        // FIRST/RECORD: running state (in/out); RECOMPUTE: checkpoint (in)
    uint8_t *o_state;
    float *U_out;          // [R][B*H*W*N] or null
    uint16_t *Po_out;      // [R][B*PH*PW*N] bf16
    float *ckU;            // FIRST: checkpoint slot (after row 0) or null
    uint8_t *cko;
    int ck_every;          // >0: rows r % ck_every == 0 write checkpoint slot r / ck_every, ck_stride elements
    long long ck_stride;   // apart (several segments per launch); 0: row 0 only
    unsigned *s_part;      // SAM partials [T][32] of this layer's spikes, or null
    unsigned *s_part_in;   // SAM partials [T][32] of the input spikes (l = 0), or null
    double *u2_part;       // l2-trace SAM: sum of U^2 per row into [T][32] fp64 partials, or null
    float *dbg_U;
    uint8_t *dbg_o;
    uint16_t *xg_out;      // or null: also write the bf16 im2col rows [R][B*H*W][32] (weight-gradient operand)
    int state_tm;          // 1: U_state / o_state / ckU / cko in the kernel's thread-major layout
                           // (layer0_state_count elements: [tile][channel chunk][c/4][tile row][4]), 0: NHWC
};
bool layer0_supported(int B, int H, int W, int C0, int N, int pool);
long long layer0_state_count(int B, int H, int W, int N, int pool);

// Fused layer-0 backward (layer0.cu): Eq.2 reverse scan + weight gradient on the tensor cores.
struct L0BwdArgs {
    const uint8_t *x;
    int T, B, H, W, C0;
    const int *row_t;      // absolute t per row (device) or null -> r
    int R;
    const float *U;        // [R][B*H*W*N] stored membranes
    const float *g;        // [R][B*PH*PW*N] gradient wrt the (pooled) output
    float *carry;          // [B*H*W*N] in/out
    float *dW;             // [N][32] fp32, accumulated (k = (dy*3+dx)*C0 + ci)
    int N, pool;
    float lam, theta;
    int surr;
    float gamma;
};
bool layer0_bwd_supported(int B, int H, int W, int C0, int N, int pool);
cudaError_t launch_layer0_bwd(const L0BwdArgs &a, cudaStream_t s, int num_sms);
cudaError_t launch_layer0_fwd(const L0FwdArgs &a, cudaStream_t s, int num_sms);

// Readout integrator + softmax cross-entropy (reading 5) and its gradients.
cudaError_t launch_readout_loss(const uint16_t *WbL, const float *cnt, const int *labels, float *z, float *dz,
                                float *loss, float *g_last, int B, int D, int K, float invT, float invBg,
                                cudaStream_t s);
cudaError_t launch_readout_wgrad(const float *dz, const float *cnt_kept, float *dWL, int B, int D, int K,
                                 float invT, cudaStream_t s, int accumulate = 0);

// Adam + bf16 shadow; transposed bf16 shadow for the dgrad GEMMs.
cudaError_t launch_adam(float *w, const float *g, float *m, float *v, uint16_t *wb, size_t n, float lr, float b1,
                        float b2, float eps, float bc1, float bc2_sqrt, cudaStream_t s);
cudaError_t launch_cast_bf16(const float *w, uint16_t *wb, size_t n, cudaStream_t s);
// dst[c][t][a] = src[a][t][c]   (src viewed [A][Tp][Cc])
cudaError_t launch_transpose_bf16(const uint16_t *src, uint16_t *dst, int A, int Tp, int Cc, cudaStream_t s);

}  // namespace sk
