/*
 * skipper_kernels.h - kernel-level entry points of the sm_100a library, for
 * per-kernel parity tests and micro-benchmarks.  They launch exactly the
 * kernels skipper_step uses (same launchers), stream-ordered on `stream`.
 * All pointers are device pointers; bf16 tensors are passed as uint16 bit
 * patterns.  Return value: a skipper_status (0 = OK); on a CUDA error the
 * message is in skipper_last_error(NULL).
 *
 * Contractions (the synaptic GEMMs of Eq.1 forward and Eq.2 backward),
 * all bf16 x bf16 -> fp32 on the tcgen05 tensor cores:
 *   fc_fwd     C[M][N]  = A[M][K] . B[N][K]^T                 (I = P(o) W^T; dgrad g = delta Wt^T)
 *   fc_wgrad   dW[N][K] (+)= D[M][N]^T . X[M][K]              (dW = sum_rows delta^T a)
 *   conv_fwd   Y[nb,y,x,co] = sum_{dy,dx,ci} Wk[co][dy*3+dx][ci] X[nb,y+dy-1,x+dx-1,ci]   (pad 1)
 *   conv_dgrad G[nb,y,x,ci] = sum_{dy,dx,co} Wt[ci][dy*3+dx][co] D[nb,y-dy+1,x-dx+1,co]
 *   conv_wgrad dW[co][dy*3+dx][ci] (+)= sum_{nb,y,x} D[nb,y,x,co] X[nb,y+dy-1,x+dx-1,ci]
 * Shape limits: K, N, cin, cout multiples of 8 (16-byte rows); conv h*w*... see DESIGN.md.
 */
#ifndef SKIPPER_KERNELS_H
#define SKIPPER_KERNELS_H

#ifdef __cplusplus
extern "C" {
#endif

int skipper_k_fc_fwd(const unsigned short *A, const unsigned short *B, float *C,
                     int M, int N, int K, void *stream);
int skipper_k_fc_wgrad(const unsigned short *D, const unsigned short *X, float *dW,
                       int M, int N, int K, int accumulate, void *stream);
int skipper_k_conv_fwd(const unsigned short *X, const unsigned short *Wk, float *Y,
                       int nb, int h, int w, int cin, int cout, void *stream);
int skipper_k_conv_dgrad(const unsigned short *D, const unsigned short *Wt, float *G,
                         int nb, int h, int w, int cin, int cout, void *stream);
int skipper_k_conv_wgrad(const unsigned short *D, const unsigned short *X, float *dW,
                         int nb, int h, int w, int cin, int cout, int accumulate, void *stream);
/* Weight gradient of a narrow-channel 3x3 conv (cin in {16, 32}, cout in {16, 32, 64}, stride 1 or 2,
 * pad 1; the ResNet-DVS layers of cfg 4), Eq.2's weight term without a column buffer:
 *   dW[co][dy*3+dx][ci] (+)= sum_{nb,y,x} D[nb,y,x,co] X[nb, s*y+dy-1, s*x+dx-1, ci]
 * D [nb][h][w][cout] and X [nb][s*h][s*w][cin] bf16 device pointers, dW [cout][9][cin] fp32 device
 * (zeroed first unless accumulate).  w must be a multiple of 16 dividing 128 and h a multiple of
 * min(h, 128 / w).  fp32 atomics: the summation order is not fixed (rounding-level differences).
 * EUNSUPPORTED for other shapes, ECUDA on a launch error. */
int skipper_k_narrow_wgrad(const unsigned short *D, const unsigned short *X, float *dW, int nb, int h, int w,
                           int cin, int cout, int stride, int accumulate, void *stream);
/* dgrad of a narrow-channel 3x3 conv (pad 1, stride s in {1, 2}), Eq.2's g term:
 *   G[nb,yi,xi,ci] = sum_{dy,dx,co} Wt[ci][dy*3+dx][co] D[nb, (yi+1-dy)/s, (xi+1-dx)/s, co]
 * (terms whose offsets are not multiples of s vanish).  h x w is the OUTPUT (delta) size: D [nb][h][w][cout]
 * and Wt [cin][9][cout] bf16, G [nb][s*h][s*w][cin] fp32 (overwritten), device pointers.  cin 16 with
 * cout 16 / 32, or cin 32 with cout 16 / 32 (64 at s = 2); s*w a multiple of 16 dividing 128.
 * EUNSUPPORTED for other shapes, ECUDA on a launch error. */
int skipper_k_narrow_dgrad(const unsigned short *D, const unsigned short *Wt, float *G, int nb, int h, int w,
                           int cin, int cout, int stride, void *stream);
/* Strided / narrow-channel implicit conv (ResNet layers, reading 8):
 *   Y[nb,y,x,co] = sum_{dy,dx,ci} Wk[co][dy*3+dx][ci] X[nb, s*y+dy-1, s*x+dx-1, ci]   (pad 1, stride s)
 * h x w is the OUTPUT size, X is [nb][s*h][s*w][cin]; cin in {16, 32} (one 32B/64B-swizzled TMA box per
 * tap) or a multiple of 64; s in {1, 2} (TMA element strides).  With sign = -1 (stride 1 only) it is the
 * dgrad of conv_dgrad above (X = D, Wk = Wt, cin = the layer's cout).  EUNSUPPORTED otherwise. */
int skipper_k_conv_s(const unsigned short *X, const unsigned short *Wk, float *Y, int nb, int h, int w, int cin,
                     int cout, int sign, int stride, void *stream);

/* The same contraction as skipper_k_conv_s for narrow channels with a cp.async gather producer (the 9 taps
 * re-read through L1; no 32-byte TMA box rows): cin in {16, 32, 48, 64}, cout a multiple of 16 up to 128. */
int skipper_k_conv_narrow(const unsigned short *X, const unsigned short *Wk, float *Y, int nb, int h, int w, int cin,
                          int cout, int sign, int stride, void *stream);

/* Fused 3x3 convolution + LIF over R timestep rows (Eq.1): for r = 0..R-1
 *   I_r = conv_fwd(X_r, Wk)  (bf16 x bf16 -> fp32, tensor cores, never written to memory)
 *   U_r = ((lam * U_{r-1}) + I_r) - theta * o_{r-1},   o_r = [U_r > theta]
 * X [R][nb][h][w][cin] bf16 (nb = batch), Wk [cout][9][cin] bf16.  U_state [nb*h*w*cout] fp32 and
 * o_state (uint8) hold (U_{-1}, o_{-1}) on entry and (U_{R-1}, o_{R-1}) on return.  Outputs:
 * P [R][nb][h'][w'][cout] bf16 spikes (pool = 1: 2x2 average, h' = h/2), U_out [R][nb*h*w*cout] fp32
 * (may be NULL).  Limits: cin % 64 == 0, cout 64 or a multiple of 128, 128 % w == 0 and the 128-pixel
 * tile covering whole image rows.  EUNSUPPORTED otherwise. */
int skipper_k_conv_lif(const unsigned short *X, const unsigned short *Wk, float *U_state, unsigned char *o_state,
                       unsigned short *P, float *U_out, int R, int nb, int h, int w, int cin, int cout, int pool,
                       float lam, float theta, void *stream);

/* Number of SMs the persistent kernels size their grids for (148 on B200). */
int skipper_k_num_sms(void);

#ifdef __cplusplus
}
#endif
#endif
