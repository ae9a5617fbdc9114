// gemm.h - host-side description of one synaptic contraction on the tcgen05 tensor cores.
//
// The synaptic GEMMs of Eq.1 (I = W o) and Eq.2 (W^T delta and
// sum_t delta o^T), layer-major over all (kept) timesteps of a segment:
// the M dimension is (t, b, h, w), so T*L tiny per-step products become L GEMMs.
#pragma once
#include <cstdint>
#include <cuda.h>
#include <cuda_runtime.h>

namespace sk {

enum OperandKind {
    OP_K2D = 0,     // K-major 2D matrix [rows][K], TMA box {64, rows}
    OP_KCONV = 1,   // K-major implicit im2col of an NHWC image, one 3x3 tap per K block
    OP_MN2D = 2,    // MN-major 2D matrix [K rows][MN], TMA boxes {64, 64}
    OP_MNCONV = 3,  // MN-major shifted NHWC image (wgrad input operand), boxes {64, W, bh, bn}
    OP_MNSHIFT = 4, // MN-major shifted NHWC image as 2D boxes of the flattened pixels at row offset
                    // dy*W + dx; rows whose shifted pixel leaves the image are zeroed in smem by the
                    // MMA warp before the MMA reads them (4D boxes measured ~2x slower through TMA)
};

// OVERWRITE: plain store; ATOMIC_ADD: TMA reduce-add (unsplit weight gradients accumulating over the
// segments: one writer per element per launch, launches in stream order -> deterministic);
// SPLIT: split s stores its partial sum into slice s of [splits][M][N] (summed in fixed order by the
// consuming scan - deterministic split-K for the forward / dgrad GEMMs);
// SLICE_ADD: split s reduce-adds into slice s of [slices][M][N] (split-K weight gradients: every slice has
// one writer per launch and the launches are stream-ordered, so each slice accumulates the segments in a
// fixed order; launch_reduce_slices sums the slices in slice order - deterministic split-K wgrad).
enum StoreMode { STORE_OVERWRITE = 0, STORE_ATOMIC_ADD = 1, STORE_SPLIT = 2, STORE_SLICE_ADD = 3 };

// Passed by value to the kernel.
struct GemmDev {
    int m_tiles, n_tiles, taps, splits;
    int num_kb, kb_per_split;
    int a_kind, b_kind;
    int conv_cb;        // channel blocks of 64 per tap (A = OP_KCONV)
    int conv_hw, conv_w;  // image H*W and W (row -> (image, y) decode)
    int conv_sign;      // +1 forward / wgrad, -1 dgrad (flipped taps)
    int cols_per_tap;   // output column offset per tap (unused when 0)
    int wg_cin;         // wgrad conv with N = (tap, cin): channels per tap (0 = N is one tap's channels)
    int transpose_out;  // the tile is D^T: TMEM lanes are output columns, TMEM columns output rows
    float *C;
    long long ldc;
    int M, N;           // valid output extent (rows, columns of one tap block)
    int store_mode;
    unsigned long long *stats;  // optional pipeline wait statistics (null in production)
    // narrow / strided implicit conv (plan_conv_s): K elements per K block (16 or 32 = one tap of a
    // 16/32-channel image, 32B/64B-swizzled boxes; 0 = the 64-element 128B-swizzled default), the conv
    // stride (TMA element strides) and the bytes one pipeline stage receives
    int kblk;
    int conv_stride;
    uint32_t stage_tx;
    int ring;               // narrow: smem ring depth (stages of stage_stride bytes)
    uint32_t stage_stride;
};

struct GemmLaunch {
    GemmDev d;
    CUtensorMap ta, tb, tc;  // operands A, B and the fp32 output
    int bn;             // 64, 128 or 256
    int mn_major;       // 0: both operands K-major; 1: both MN-major (wgrad)
    int cs = 1;         // cluster size: B tile multicast across cs CTAs working on consecutive M tiles
};

// Tensor-map builders (bf16, 128-byte swizzle, OOB -> zero).
bool make_map_2d(CUtensorMap *m, const void *ptr, uint64_t inner, uint64_t outer, uint32_t box_inner,
                 uint32_t box_outer);
bool make_map_conv(CUtensorMap *m, const void *ptr, uint64_t C, uint64_t W, uint64_t H, uint64_t NB,
                   uint32_t box_w, uint32_t box_h, uint32_t box_n);

// Plans (return false on unsupported geometry).  All pointers are device pointers.
// C[M][N] = A[M][K] . B[N][K]^T
bool plan_fc(GemmLaunch *g, const void *A, const void *B, float *C, int M, int N, int K, int splits = 1);
// dW[N][K] (+)= D[M][N]^T . X[M][K]   (reduction over the M rows).  slices > 0: dW is the slice buffer
// [slices][N][K] and split s reduce-adds into slice s (STORE_SLICE_ADD); needs fc_wgrad_splits(M) <= slices.
bool plan_fc_wgrad(GemmLaunch *g, const void *D, const void *X, float *dW, int M, int N, int K, int num_sms,
                   int slices = 0);
// split-K factor plan_fc_wgrad / plan_conv_wgrad choose for a reduction of M rows (monotone in M, so the
// value at the largest M of a layer bounds every launch of that layer)
int fc_wgrad_splits(long long M, int N, int K, int num_sms);
int conv_wgrad_splits(long long M, int cin, int cout, int num_sms);
// conv forward / dgrad: Y[nb,h,w,cout] from X[nb,h,w,cin] and Wk[cout][9][cin];
// dgrad: G[nb,h,w,cin] from D[nb,h,w,cout] and Wt[cin][9][cout]
bool plan_conv(GemmLaunch *g, const void *X, const void *Wk, float *Y, int nb, int h, int w, int cin, int cout,
               int sign);
// conv forward / dgrad with stride (1 or 2) and narrow channels (cin in {16, 32} or a multiple of 64):
// Y[nb, h, w, cout] (h x w = OUTPUT size) from X[nb, s*h, s*w, cin]; pixels on M, non-transposed.
// dgrad of a stride-1 conv: sign = -1 with D as X and Wt [cin][9][cout] as Wk (as plan_conv).
bool plan_conv_s(GemmLaunch *g, const void *X, const void *Wk, float *Y, int nb, int h, int w, int cin, int cout,
                 int sign, int stride);
// Narrow-channel conv with a cp.async gather producer (conv_narrow.cu): cin in {16, 32, 48, 64},
// cout a multiple of 16 up to 128, stride 1 or 2 (sign +1), or the stride-1 dgrad (sign -1, Wk = Wt).
struct NarrowConvArgs {
    const uint16_t *X;   // [nb][Hin][Win][Cin] bf16 (LIF: [R][nb][Hin][Win][Cin], row r read by row r)
    const uint16_t *Wk;  // [Cout][9][Cin] bf16
    float *Y;            // [nb][H][W][Cout] fp32 (conv only)
    int nb, H, W, Hin, Win, Cin, Cout, stride, sign;
    int ring;            // filled by the launcher
    // ---- fused LIF scan (launch_conv_narrow_lif): Eq.1 over the R rows of a segment in the epilogue, with
    // the same state / output / checkpoint / SAM / residual semantics as ScanFwdArgs (kernels.h), unpooled
    int R, restore, t0;
    const int *row_t;
    float *U_state;
    uint8_t *o_state;
    float *U_out;
    uint16_t *Po_out;
    float *ckU;
    uint8_t *cko;
    int ck_every;          // >0: rows r % ck_every == 0 write checkpoint slot r / ck_every (ck_stride elements
    long long ck_stride;   // apart); 0: row 0 writes slot 0 (one segment per launch)
    unsigned *s_part;
    double *u2_part;
    float *cnt;
    float *dbg_U;
    uint8_t *dbg_o;
    const uint16_t *res;
    int res_H, res_W, res_C, res_stride, res_lo;
    float lam, theta;
};
bool conv_narrow_supported(int cin, int cout, int stride, int sign);
cudaError_t launch_conv_narrow(const NarrowConvArgs &a, cudaStream_t s, int num_sms);
bool conv_narrow_lif_supported(int cin, int cout, int stride);
cudaError_t launch_conv_narrow_lif(const NarrowConvArgs &a, cudaStream_t s, int num_sms);
// The same fused conv + LIF on warp-level bf16 MMAs over staged input rows (narrow_lif.cu): cin 16,
// cout 16 / 32, stride 1 / 2, output width a multiple of 16 dividing 128
bool narrow_lif_mma_supported(int cin, int cout, int stride, int H, int W);
cudaError_t launch_narrow_lif_mma(const NarrowConvArgs &a, cudaStream_t s, int num_sms);
// conv wgrad: dW[cout][9][cin] (+)= sum D[.,cout] X_shift[.,cin]
bool plan_conv_wgrad(GemmLaunch *g, const void *D, const void *X, float *dW, int nb, int h, int w, int cin, int cout,
                     int num_sms, int slices = 0);

cudaError_t gemm_run(const GemmLaunch &g, cudaStream_t stream, int num_sms);

// Fused 3x3 convolution + LIF scan over the R rows of a segment (conv_lif.cu).  The input X is the
// previous layer's output [rows_in][B][H][W][Cin] bf16 (row r of the segment reads input row r), Wk is
// [Cout][9][Cin] bf16.  State / output pointers follow ScanFwdArgs (kernels.h); cnt is not supported.
struct ConvLifArgs {
    int B, H, W, Cin, Cout, pool;
    int R, restore, t0;
    const int *row_t;
    float *U_state;
    uint8_t *o_state;
    float *U_out;
    uint16_t *Po_out;
    float *ckU;
    uint8_t *cko;
    int ck_every;          // as NarrowConvArgs
    long long ck_stride;
    unsigned *s_part;
    double *u2_part;  // l2-trace SAM partials [T][32] or null
    float *dbg_U;
    uint8_t *dbg_o;
    float lam, theta;
    // 1: U_state / o_state / ckU / cko in the kernel's thread-major layout (conv_lif_state_count elements:
    // [unit][channel half][channel / 4][pixel of the 128-pixel tile][4]) - coalesced state loads / stores;
    // 0: NHWC [B][H][W][Cout] (the kernel-level test API)
    int state_tm;
    // filled by launch_conv_lif
    int m_tiles, n_tiles, num_kb, conv_cb;
    int stages;      // smem ring depth
    int halo_bytes;  // bytes of one halo activation box (HALO variant)
    int diag;  // SKIPPER_CL_DIAG timing experiments: 1 = no epilogue work, 2 = no MMA
    // backward (launch_conv_lif_bwd): U rows [R][B][H][W][Cout] fp32 of the layer whose delta is computed,
    // its carry [B][H][W][Cout] (delta after the last row in, delta at row 0 out), the bf16 delta rows out,
    // surrogate kind (SURR_*) and gamma
    const float *bU;
    float *bcarry;
    uint16_t *bdelta;
    int surr;
    float gamma;
};
bool conv_lif_supported(int B, int H, int W, int cin, int cout, int pool);
// elements of one state / checkpoint slot in the thread-major layout (>= B*H*W*Cout: whole 128-pixel tiles)
long long conv_lif_state_count(int B, int H, int W, int cout);
cudaError_t launch_conv_lif(const void *X, int rows_in, const void *Wk, ConvLifArgs a, cudaStream_t s, int num_sms);
// NEXT-1 backward half (K2 + K4 fused): for a stride-1 3x3 layer l with Cin = C_l (the delta operand's
// channels) and Cout = C_{l-1} (multiple of 64), g = conv(delta^l, W^l flipped) with the reverse scan of layer l-1
// in the epilogue.  D: delta^l rows [rows_in][B][H][W][Cin] bf16 (row r = kept row r), Wt: W^l as
// [Cout][9][Cin] bf16 (the dgrad layout [C_{l-1}][3][3][C_l]); writes a.bdelta rows and a.bcarry.
bool conv_lif_bwd_supported(int B, int H, int W, int cin, int cout);
cudaError_t launch_conv_lif_bwd(const void *D, int rows_in, const void *Wt, ConvLifArgs a, cudaStream_t s, int num_sms);

int device_num_sms();

}  // namespace sk
