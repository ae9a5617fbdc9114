// lif_kernels.cu - K1 (forward LIF scan), K4 (reverse surrogate scan), layer-0 input staging / SAM,
// readout + loss, Adam.  sm_100a CUDA cores; HBM-bound streams.
//
// Eq.1:  U_t = lam*U_{t-1} + W o^{l-1}_t - theta*o^l_{t-1};  o_t = [U_t > theta]
//   evaluated without FMA in the order ((lam*U) + I) - theta*o so that spikes are bit-identical to
//   the oracle.
// Eq.2:  delta^l_t = sigma'(U^l_t) * g^l_t + lam * delta^l_{t+1}, reset detached.
// Eq.4:  s_t = sum_l sum(o^l_t), accumulated in [T][32] partial counters.
#include "common.cuh"
#include "kernels.h"

#ifndef SK_FS_CH_SPLIT
#define SK_FS_CH_SPLIT 4  // rows per chunk of the fc forward scan over split-K partial currents
#endif
#ifndef SK_BS_CH_SPLIT
#define SK_BS_CH_SPLIT 4  // rows per chunk of the fc reverse scan over split-K partial gradients
#endif

namespace sk {

SK_DEV float lif_update(float U, float I, float o, float lam, float th) {
    return __fsub_rn(__fadd_rn(__fmul_rn(lam, U), I), o != 0.f ? th : 0.f);  // theta * o, o in {0, 1}: exact select
}

// sigma'(U) of reading 4; inv_th = 1 / theta computed once per thread (the reverse scan is issue-bound:
// a multiply instead of an IEEE division per neuron-step; within 1 ulp of |U - theta| / theta)
SK_DEV float surrogate(float U, float th, float inv_th, int kind, float gamma) {
    if (kind == SURR_TRIANGLE) {
        const float v = 1.0f - fabsf(U - th) * inv_th;
        return v > 0.0f ? gamma * v : 0.0f;
    }
    const float d = 1.0f + gamma * fabsf(U - th);
    return __frcp_rn(d * d);
}

SK_DEV uint2 pack_bf16x4(float a, float b, float c, float d) {
    uint2 r;
    r.x = (uint32_t)f2bf_bits(a) | ((uint32_t)f2bf_bits(b) << 16);
    r.y = (uint32_t)f2bf_bits(c) | ((uint32_t)f2bf_bits(d) << 16);
    return r;
}

SK_DEV float4 ldg4(const float *p) { return __ldg(reinterpret_cast<const float4 *>(p)); }

static constexpr int MAX_SPLIT = 8;

// Sum of the split-K partial slices in fixed order s = 0, 1, ... (deterministic, identical in the
// first pass and the recompute because the split count is a per-layer constant).  All partial
// loads are issued before the (ordered) additions.
SK_DEV float4 ldg4_split(const float *p, int nsplit, long long stride) {
    float4 w[MAX_SPLIT];
#pragma unroll
    for (int s = 0; s < MAX_SPLIT; ++s)
        w[s] = s < nsplit ? ldg4(p + s * stride) : make_float4(0.f, 0.f, 0.f, 0.f);
    float4 v = w[0];
#pragma unroll
    for (int s = 1; s < MAX_SPLIT; ++s) {
        if (s < nsplit) {
            v.x = __fadd_rn(v.x, w[s].x);
            v.y = __fadd_rn(v.y, w[s].y);
            v.z = __fadd_rn(v.z, w[s].z);
            v.w = __fadd_rn(v.w, w[s].w);
        }
    }
    return v;
}
SK_DEV float ldg_split(const float *p, int nsplit, long long stride) {
    float w[MAX_SPLIT];
#pragma unroll
    for (int s = 0; s < MAX_SPLIT; ++s) w[s] = s < nsplit ? __ldg(p + s * stride) : 0.f;
    float v = w[0];
#pragma unroll
    for (int s = 1; s < MAX_SPLIT; ++s)
        if (s < nsplit) v = __fadd_rn(v, w[s]);
    return v;
}

// ============================================================================ K1 forward scan
// One thread owns 4 consecutive channels of NP pixels (NP = 4: the 2x2 window of one pooled output).
// The currents of CH rows are loaded before the recurrence consumes them (the loads do not depend
// on the recurrence); __launch_bounds__(256, 4) keeps the register file at <= 64 per thread so
// 32 warps per SM keep enough 16-byte loads in flight for HBM.  Spike counts per row (SAM, Eq.4)
// go through shared-memory atomics and one global atomic per row per block at the end.
template <int POOL, int SPLIT>
__global__ void __launch_bounds__(256, POOL ? 3 : 4) lif_fwd_kernel(const ScanFwdArgs a) {
    pdl_enter();
    constexpr int NP = POOL ? 4 : 1;
    constexpr int CH = POOL ? 2 : (SPLIT ? 4 : 8);
    extern __shared__ unsigned s_cnt[];  // [R] block spike count per row (when a.s_part)
    const int C = a.C;
    const int C4 = C >> 2;
    const long long HW = (long long)a.H * a.W;
    const long long P = POOL ? (long long)a.B * (a.H / 2) * (a.W / 2) * C4 : (long long)a.B * HW * C4;
    const long long p = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    const bool active = p < P;
    const long long rs = (long long)a.B * HW * C;  // neurons per row
    const long long ors = POOL ? rs / 4 : rs;       // outputs per row
    const int nspl = SPLIT ? a.nsplit : 1;

    if (a.s_part) {
        for (int r = threadIdx.x; r < a.R; r += blockDim.x) s_cnt[r] = 0;
        __syncthreads();
    }
    int nidx[NP], oidx = 0;  // offsets within one row (a row holds < 2^31 neurons)
    {
        const long long pp = active ? p : 0;
        const int c4 = (int)(pp % C4);
        long long rest = pp / C4;
        if (POOL) {
            const int PW = a.W / 2, PH = a.H / 2;
            const int px = (int)(rest % PW);
            rest /= PW;
            const int py = (int)(rest % PH);
            const long long b = rest / PH;
#pragma unroll
            for (int k = 0; k < NP; ++k)
                nidx[k] = (int)(((b * a.H + 2 * py + (k >> 1)) * a.W + 2 * px + (k & 1)) * C + 4 * c4);
            oidx = (int)(((b * PH + py) * PW + px) * C + 4 * c4);
        } else {
            nidx[0] = (int)(rest * C + 4 * c4);
            oidx = nidx[0];
        }
    }
    // residual shortcut (reading 8): offset of this thread's 4 channels in a source row, or -1 (zero pad)
    long long res_off = -1, res_rs = 0;
    if (!POOL && a.res && active) {
        const long long pix = p / C4;
        const int x = (int)(pix % a.W), y = (int)((pix / a.W) % a.H);
        const long long b = pix / HW;
        const int cs = 4 * (int)(p % C4) - a.res_lo;
        res_rs = (long long)a.B * a.res_H * a.res_W * a.res_C;
        if (cs >= 0 && cs < a.res_C)
            res_off = ((b * a.res_H + (long long)y * a.res_stride) * a.res_W + (long long)x * a.res_stride) * a.res_C + cs;
    }

    float U[NP][4];
    uint32_t ob = 0;  // spike bits, bit 4k+i
    if (active) {
#pragma unroll
        for (int k = 0; k < NP; ++k) {
            const float4 u = *reinterpret_cast<const float4 *>(a.U_state + nidx[k]);
            const uchar4 o4 = *reinterpret_cast<const uchar4 *>(a.o_state + nidx[k]);
            U[k][0] = u.x; U[k][1] = u.y; U[k][2] = u.z; U[k][3] = u.w;
            ob |= (o4.x ? 1u : 0u) << (4 * k) | (o4.y ? 1u : 0u) << (4 * k + 1) |
                  (o4.z ? 1u : 0u) << (4 * k + 2) | (o4.w ? 1u : 0u) << (4 * k + 3);
        }
    } else {
#pragma unroll
        for (int k = 0; k < NP; ++k) U[k][0] = U[k][1] = U[k][2] = U[k][3] = 0.f;
    }
    float cacc[4] = {0.f, 0.f, 0.f, 0.f};
    auto bit = [&](int k, int i) { return (float)((ob >> (4 * k + i)) & 1u); };

    auto emit_row = [&](int r) {  // outputs of row r from the current (U, spikes)
        float out[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            float sum = 0.f;
#pragma unroll
            for (int k = 0; k < NP; ++k) sum += bit(k, i);
            out[i] = POOL ? sum * 0.25f : sum;
            cacc[i] += out[i];
        }
        *reinterpret_cast<uint2 *>(a.Po_out + (long long)r * ors + oidx) = pack_bf16x4(out[0], out[1], out[2], out[3]);
        if (a.U_out) {
#pragma unroll
            for (int k = 0; k < NP; ++k)
                *reinterpret_cast<float4 *>(a.U_out + (long long)r * rs + nidx[k]) =
                    make_float4(U[k][0], U[k][1], U[k][2], U[k][3]);
        }
        if (a.dbg_U) {
            const long long t = a.row_t ? a.row_t[r] : a.t0 + r;
#pragma unroll
            for (int k = 0; k < NP; ++k) {
                *reinterpret_cast<float4 *>(a.dbg_U + t * rs + nidx[k]) = make_float4(U[k][0], U[k][1], U[k][2], U[k][3]);
                *reinterpret_cast<uchar4 *>(a.dbg_o + t * rs + nidx[k]) =
                    make_uchar4((unsigned char)bit(k, 0), (unsigned char)bit(k, 1), (unsigned char)bit(k, 2),
                                (unsigned char)bit(k, 3));
            }
        }
    };

    int r0 = 0;
    if (a.restore) {
        if (active) emit_row(0);
        r0 = 1;
    }
    const int lane = threadIdx.x & 31;
    for (int rb = r0; rb < a.R; rb += CH) {
        float4 Iv[CH][NP];
#pragma unroll
        for (int j = 0; j < CH; ++j) {
            const int r = rb + j;
#pragma unroll
            for (int k = 0; k < NP; ++k) {
                if (active && r < a.R) {
                    const float *src = a.I + (long long)r * rs + nidx[k];
                    Iv[j][k] = SPLIT ? ldg4_split(src, nspl, a.split_stride) : ldg4(src);
                    if (!POOL && res_off >= 0) {  // I += S(a^r): exact (spikes added to the fp32 GEMM sum)
                        const uint2 rv = __ldg(reinterpret_cast<const uint2 *>(a.res + (long long)r * res_rs + res_off));
                        Iv[j][k].x = __fadd_rn(Iv[j][k].x, __uint_as_float(rv.x << 16));
                        Iv[j][k].y = __fadd_rn(Iv[j][k].y, __uint_as_float(rv.x & 0xffff0000u));
                        Iv[j][k].z = __fadd_rn(Iv[j][k].z, __uint_as_float(rv.y << 16));
                        Iv[j][k].w = __fadd_rn(Iv[j][k].w, __uint_as_float(rv.y & 0xffff0000u));
                    }
                } else {
                    Iv[j][k] = make_float4(0.f, 0.f, 0.f, 0.f);
                }
            }
        }
#pragma unroll
        for (int j = 0; j < CH; ++j) {
            const int r = rb + j;
            if (r >= a.R) break;  // block-uniform
            unsigned nspk = 0;
            double q2 = 0.0;
            if (active) {
                uint32_t nb = 0;
#pragma unroll
                for (int k = 0; k < NP; ++k) {
                    const float Ii[4] = {Iv[j][k].x, Iv[j][k].y, Iv[j][k].z, Iv[j][k].w};
#pragma unroll
                    for (int i = 0; i < 4; ++i) {
                        U[k][i] = lif_update(U[k][i], Ii[i], bit(k, i), a.lam, a.theta);
                        nb |= (U[k][i] > a.theta ? 1u : 0u) << (4 * k + i);
                        if (a.u2_part) q2 += (double)U[k][i] * (double)U[k][i];
                    }
                }
                ob = nb;
                nspk = __popc(ob);
                emit_row(r);
                if (a.ckU && (a.ck_every ? r % a.ck_every == 0 : r == 0)) {
                    const long long slot = a.ck_every ? (long long)(r / a.ck_every) * rs : 0;
#pragma unroll
                    for (int k = 0; k < NP; ++k) {
                        *reinterpret_cast<float4 *>(a.ckU + slot + nidx[k]) = make_float4(U[k][0], U[k][1], U[k][2], U[k][3]);
                        *reinterpret_cast<uchar4 *>(a.cko + slot + nidx[k]) =
                            make_uchar4((unsigned char)bit(k, 0), (unsigned char)bit(k, 1), (unsigned char)bit(k, 2),
                                        (unsigned char)bit(k, 3));
                    }
                }
            }
            if (a.s_part) {
                const unsigned v = __reduce_add_sync(0xffffffffu, nspk);
                if (lane == 0 && v) atomicAdd(&s_cnt[r], v);
            }
            if (a.u2_part) u2_warp_add(a.u2_part, a.row_t ? a.row_t[r] : a.t0 + r, q2);
        }
    }
    if (active) {
        if (!a.restore) {
#pragma unroll
            for (int k = 0; k < NP; ++k) {
                *reinterpret_cast<float4 *>(a.U_state + nidx[k]) = make_float4(U[k][0], U[k][1], U[k][2], U[k][3]);
                *reinterpret_cast<uchar4 *>(a.o_state + nidx[k]) =
                    make_uchar4((unsigned char)bit(k, 0), (unsigned char)bit(k, 1), (unsigned char)bit(k, 2),
                                (unsigned char)bit(k, 3));
            }
        }
        if (a.cnt) {
            float4 *cp = reinterpret_cast<float4 *>(a.cnt + oidx);
            float4 cv = *cp;
            cv.x += cacc[0]; cv.y += cacc[1]; cv.z += cacc[2]; cv.w += cacc[3];
            *cp = cv;
        }
    }
    if (a.s_part) {
        __syncthreads();
        for (int r = threadIdx.x; r < a.R; r += blockDim.x) {
            const unsigned v = s_cnt[r];
            const long long t = a.row_t ? a.row_t[r] : a.t0 + r;
            if (v) atomicAdd(a.s_part + t * 32 + (blockIdx.x & 31), v);
        }
    }
}

// Small unpooled layers (fc): one thread per neuron so that a 64k-neuron row still fills the GPU;
// the split-K partial currents of CH rows are all in flight before the recurrence consumes them.
template <int CH, int SPLIT>
__global__ void __launch_bounds__(256) lif_fwd_small_kernel(const ScanFwdArgs a) {
    pdl_enter();
    if (sk_pdl_early()) pdl_trigger();
    extern __shared__ unsigned s_cnt[];
    const long long rs = (long long)a.B * a.H * a.W * a.C;
    const long long n = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    const bool active = n < rs;
    if (a.s_part) {
        for (int r = threadIdx.x; r < a.R; r += blockDim.x) s_cnt[r] = 0;
        __syncthreads();
    }
    float U = active ? a.U_state[n] : 0.f;
    float o = (active && a.o_state[n]) ? 1.f : 0.f;
    float cacc = 0.f;
    auto emit = [&](int r) {
        a.Po_out[(long long)r * rs + n] = o != 0.f ? (uint16_t)0x3F80 : (uint16_t)0;
        cacc += o;
        if (a.U_out) a.U_out[(long long)r * rs + n] = U;
        if (a.dbg_U) {
            const long long t = a.row_t ? a.row_t[r] : a.t0 + r;
            a.dbg_U[t * rs + n] = U;
            a.dbg_o[t * rs + n] = o != 0.f ? 1 : 0;
        }
    };
    int r0 = 0;
    if (a.restore) {
        if (active) emit(0);
        r0 = 1;
    }
    const int lane = threadIdx.x & 31;
    // two chunks of CH rows in flight: the loads of chunk k+1 are issued before the recurrence of chunk k
    auto load = [&](float (&Iv)[CH], int rb) {
#pragma unroll
        for (int j = 0; j < CH; ++j) {
            const int r = rb + j;
            const float *src = a.I + (long long)r * rs + n;
            Iv[j] = (active && r < a.R) ? (SPLIT ? ldg_split(src, a.nsplit, a.split_stride) : __ldg(src)) : 0.f;
        }
    };
    auto consume = [&](const float (&Iv)[CH], int rb) {
#pragma unroll
        for (int j = 0; j < CH; ++j) {
            const int r = rb + j;
            if (r >= a.R) break;
            unsigned spk = 0;
            double q2 = 0.0;
            if (active) {
                U = lif_update(U, Iv[j], o, a.lam, a.theta);
                q2 = (double)U * (double)U;
                o = U > a.theta ? 1.f : 0.f;
                spk = o != 0.f ? 1u : 0u;
                emit(r);
                if (a.ckU && (a.ck_every ? r % a.ck_every == 0 : r == 0)) {
                    const long long slot = a.ck_every ? (long long)(r / a.ck_every) * rs : 0;
                    a.ckU[slot + n] = U;
                    a.cko[slot + n] = (uint8_t)spk;
                }
            }
            if (a.s_part) {
                const unsigned v = __reduce_add_sync(0xffffffffu, spk);
                if (lane == 0 && v) atomicAdd(&s_cnt[r], v);
            }
            if (a.u2_part) u2_warp_add(a.u2_part, a.row_t ? a.row_t[r] : a.t0 + r, q2);
        }
    };
    {
        float IA[CH], IB[CH];
        int rb = r0;
        if (rb < a.R) load(IA, rb);
        while (rb < a.R) {
            if (rb + CH < a.R) load(IB, rb + CH);
            consume(IA, rb);
            rb += CH;
            if (rb >= a.R) break;
            if (rb + CH < a.R) load(IA, rb + CH);
            consume(IB, rb);
            rb += CH;
        }
    }
    if (active) {
        if (!a.restore) {
            a.U_state[n] = U;
            a.o_state[n] = o != 0.f ? 1 : 0;
        }
        if (a.cnt) a.cnt[n] += cacc;
    }
    if (a.s_part) {
        __syncthreads();
        for (int r = threadIdx.x; r < a.R; r += blockDim.x) {
            const unsigned v = s_cnt[r];
            const long long t = a.row_t ? a.row_t[r] : a.t0 + r;
            if (v) atomicAdd(a.s_part + t * 32 + (blockIdx.x & 31), v);
        }
    }
}

cudaError_t launch_lif_fwd(const ScanFwdArgs &a, cudaStream_t s) {
    if (a.C % 4) return cudaErrorInvalidValue;
    if (a.res && (a.pool || a.H * a.W == 1 || a.res_C % 4 || a.res_lo % 4 || a.res_stride < 1)) return cudaErrorInvalidValue;
    // fc layers too small for 4 neurons per thread to fill the GPU (2 blocks of 256 per SM) run one neuron
    // per thread; larger ones (VGG-11 fc4096 x B=128 over T=200 rows) take the vectorised kernel: the
    // per-row overhead (SAM reduction, checkpoint test) is amortised over 4 neurons (cfg 3: the two
    // 524-us fc-tail scans of the first pass drop by ~400 us together)
    if (!a.pool && !a.res && a.H * a.W == 1 && (long long)a.B * a.C < 4LL * 2 * 148 * 256) {
        const long long rs = (long long)a.B * a.C;
        const size_t smem = a.s_part ? (size_t)a.R * sizeof(unsigned) : 0;
        if (smem > 48 * 1024) return cudaErrorInvalidValue;
        if (a.nsplit > 1)
            sk_launch(lif_fwd_small_kernel<SK_FS_CH_SPLIT, 1>, (unsigned)((rs + 255) / 256), 256, smem, s, a);
        else
            sk_launch(lif_fwd_small_kernel<8, 0>, (unsigned)((rs + 255) / 256), 256, smem, s, a);
        return cudaGetLastError();
    }
    const long long HW = (long long)a.H * a.W;
    const long long P = a.pool ? (long long)a.B * (a.H / 2) * (a.W / 2) * (a.C / 4) : (long long)a.B * HW * (a.C / 4);
    const int threads = 256;
    const long long blocks = (P + threads - 1) / threads;
    if (blocks == 0) return cudaSuccess;
    const size_t smem = a.s_part ? (size_t)a.R * sizeof(unsigned) : 0;
    if (smem > 48 * 1024) return cudaErrorInvalidValue;
    const bool split = a.nsplit > 1;
    if (a.pool) {
        if (split) sk_launch(lif_fwd_kernel<1, 1>, (unsigned)blocks, threads, smem, s, a);
        else sk_launch(lif_fwd_kernel<1, 0>, (unsigned)blocks, threads, smem, s, a);
    } else {
        if (split) sk_launch(lif_fwd_kernel<0, 1>, (unsigned)blocks, threads, smem, s, a);
        else sk_launch(lif_fwd_kernel<0, 0>, (unsigned)blocks, threads, smem, s, a);
    }
    return cudaGetLastError();
}

// ============================================================================ K4 reverse scan
// One thread owns 4 neurons (a float4 of channels of one pixel) and walks the rows downwards:
//     delta_r = sigma'(U_r) * (gs * g_r) + lam * delta_{r+1}          (Eq.2, carry = delta after the last row)
// The loop body is lean on purpose - the round-1 version was issue-bound (ncu: 80 % issue slots, 315 warp
// instructions per row, a third of them 64-bit address arithmetic, branches and local-memory spills of
// the prefetch arrays): row pointers walk down by a per-row stride, the surrogate kind is a template
// parameter, gs * gamma is folded, and rows are consumed in unrolled chunks of CH with a scalar tail.
#ifndef SK_BWD_CH
#define SK_BWD_CH 2
#endif
#ifndef SK_BWD_MINB
#define SK_BWD_MINB 8
#endif
#ifndef SK_BWD_CH1_MAX_R
#define SK_BWD_CH1_MAX_R 12
#endif
template <int SPLIT, int KIND, int CH>
__global__ void __launch_bounds__(256, SPLIT ? 4 : SK_BWD_MINB) lif_bwd_kernel(const ScanBwdArgs a) {
    pdl_enter();
    const int C = a.C;
    const long long HW = (long long)a.H * a.W;
    const long long rs = (long long)a.B * HW * C;
    const long long P = rs / 4;
    const long long p = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (p >= P) return;
    const long long n0 = 4 * p;
    long long gi = n0, grs = rs;
    if (a.g_pooled) {
        const int c = (int)(n0 % C);
        const long long pixel = n0 / C;
        const int x = (int)(pixel % a.W);
        const int y = (int)((pixel / a.W) % a.H);
        const long long b = pixel / HW;
        gi = ((b * (a.H / 2) + y / 2) * (a.W / 2) + x / 2) * C + c;
        grs = rs / 4;
    }
    if (a.g_broadcast) grs = 0;
    const float gs = a.g_pooled ? 0.25f : 1.0f;
    const int nspl = SPLIT ? a.nsplit : 1;
    // shortcut source (reading 8): S^T(delta of the receiving layer) joins g at this neuron, or not
    const uint2 *rdp = nullptr;
    long long rd_rs = 0;
    if (a.res_delta) {
        const int c = (int)(n0 % C);
        const long long pixel = n0 / C;
        const int x = (int)(pixel % a.W), y = (int)((pixel / a.W) % a.H);
        const long long b = pixel / HW;
        const int sr = a.res_stride, Hr = a.H / sr, Wr = a.W / sr;
        rd_rs = (long long)a.B * Hr * Wr * a.res_C;
        if (y % sr == 0 && x % sr == 0)
            rdp = reinterpret_cast<const uint2 *>(a.res_delta + ((b * Hr + y / sr) * Wr + x / sr) * a.res_C + c + a.res_lo);
    }
    const float th = a.theta, inv_th = 1.0f / a.theta, lam = a.lam;
    const float ggs = a.gamma * gs;  // triangle: gs * sigma' = (gs * gamma) * max(0, 1 - |U - theta| / theta)
    auto sgm = [&](float u) -> float {  // gs * sigma'(u), reading 4
        if (KIND == SURR_TRIANGLE) return ggs * fmaxf(0.0f, 1.0f - fabsf(u - th) * inv_th);
        const float dd = 1.0f + a.gamma * fabsf(u - th);
        return gs * __frcp_rn(dd * dd);
    };
    int r = a.R - 1;
    const float *Up = a.U + (long long)r * rs + n0;
    const float *Gp = a.g + (long long)r * grs + gi;
    uint2 *Dp = a.delta ? reinterpret_cast<uint2 *>(a.delta + (long long)r * rs + n0) : nullptr;
    const uint2 *Rp = rdp ? rdp + (long long)r * (rd_rs / 4) : nullptr;
    const long long rs4 = rs / 4, rd4 = rd_rs / 4;   // uint2 = 4 bf16
    float4 d = *reinterpret_cast<const float4 *>(a.carry + n0);
    auto load_g = [&](const float *gp, const uint2 *rp) -> float4 {
        float4 g = SPLIT ? ldg4_split(gp, nspl, a.split_stride) : ldg4(gp);
        if (rp) {  // unpooled layers only: gs = 1
            const uint2 rv = __ldg(rp);
            g.x = __fadd_rn(g.x, __uint_as_float(rv.x << 16));
            g.y = __fadd_rn(g.y, __uint_as_float(rv.x & 0xffff0000u));
            g.z = __fadd_rn(g.z, __uint_as_float(rv.y << 16));
            g.w = __fadd_rn(g.w, __uint_as_float(rv.y & 0xffff0000u));
        }
        return g;
    };
    auto step = [&](const float4 &u, const float4 &g, uint2 *dp) {
        d.x = sgm(u.x) * g.x + lam * d.x;
        d.y = sgm(u.y) * g.y + lam * d.y;
        d.z = sgm(u.z) * g.z + lam * d.z;
        d.w = sgm(u.w) * g.w + lam * d.w;
        if (dp) *dp = pack_bf16x4(d.x, d.y, d.z, d.w);
    };
    for (; r >= CH - 1; r -= CH) {
        float4 uv[CH], gv[CH];
#pragma unroll
        for (int j = 0; j < CH; ++j) {
            uv[j] = ldg4(Up - j * rs);
            gv[j] = load_g(Gp - j * grs, Rp ? Rp - j * rd4 : nullptr);
        }
#pragma unroll
        for (int j = 0; j < CH; ++j) step(uv[j], gv[j], Dp ? Dp - j * rs4 : nullptr);
        Up -= CH * rs;
        Gp -= CH * grs;
        if (Dp) Dp -= CH * rs4;
        if (Rp) Rp -= CH * rd4;
    }
    for (; r >= 0; --r) {
        step(ldg4(Up), load_g(Gp, Rp), Dp);
        Up -= rs;
        Gp -= grs;
        if (Dp) Dp -= rs4;
        if (Rp) Rp -= rd4;
    }
    *reinterpret_cast<float4 *>(a.carry + n0) = d;
}

// Small unpooled layers (fc): one thread per neuron (see lif_fwd_small_kernel).
template <int CH, int SPLIT>
__global__ void __launch_bounds__(256) lif_bwd_small_kernel(const ScanBwdArgs a) {
    pdl_enter();
    if (sk_pdl_early()) pdl_trigger();
    const long long rs = (long long)a.B * a.C;
    const long long n = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (n >= rs) return;
    const long long grs = a.g_broadcast ? 0 : rs;
    const float inv_th = 1.0f / a.theta;
    float d = a.carry[n];
    for (int rb = a.R - 1; rb >= 0; rb -= CH) {
        float gv[CH], uv[CH];
#pragma unroll
        for (int j = 0; j < CH; ++j) {
            const int r = rb - j;
            gv[j] = uv[j] = 0.f;
            if (r >= 0) {
                const float *src = a.g + (long long)r * grs + n;
                gv[j] = SPLIT ? ldg_split(src, a.nsplit, a.split_stride) : __ldg(src);
                uv[j] = __ldg(a.U + (long long)r * rs + n);
            }
        }
#pragma unroll
        for (int j = 0; j < CH; ++j) {
            const int r = rb - j;
            if (r >= 0) {
                d = surrogate(uv[j], a.theta, inv_th, a.surr, a.gamma) * gv[j] + a.lam * d;
                if (a.delta) a.delta[(long long)r * rs + n] = f2bf_bits(d);
            }
        }
    }
    a.carry[n] = d;
}

// fc layers with long row ranges (FULL / CKPT / TBPTT segments): Eq.2's reverse recurrence is affine in delta,
//     delta_r = c_r + lam * delta_{r+1},   c_r = sigma'(U_r) g_r,
// so a segment of rows maps the delta after it to the delta at its first row by (A, Bv) = (lam^len, sum_k
// lam^(k - lo) c_k), and segments compose.  A warp holds 8 neurons x 4 row chunks (lane = chunk * 8 +
// neuron, so each row's 8 neurons are one 32-byte sector): every lane folds its chunk to (A, Bv), the four
// chunk maps of a neuron are exchanged with __shfl_sync and composed from the carry down to chunk 0, and
// each lane re-walks its chunk from its exact incoming delta, writing delta_r - the serial depth drops from
// R to R/4 + 4.  (Rounding differs from the serial walk only in the composed incoming deltas.)
template <int SPLIT, int KIND>
__global__ void __launch_bounds__(256) lif_bwd_warp_kernel(const ScanBwdArgs a) {
    pdl_enter();
    if (sk_pdl_early()) pdl_trigger();
    constexpr int NCH = 4, NPW = 32 / NCH;   // row chunks, neurons per warp
    const long long rs = (long long)a.B * a.C;
    const int lane = threadIdx.x & 31, q = lane % NPW, j = lane / NPW;
    const long long warp = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const long long n = warp * NPW + q;
    const bool act = n < rs;
    const long long nn = act ? n : 0;
    const long long grs = a.g_broadcast ? 0 : rs;
    const float th = a.theta, inv_th = 1.0f / a.theta, lam = a.lam;
    auto c_at = [&](int r) -> float {  // sigma'(U_r) g_r
        const float *gp = a.g + (long long)r * grs + nn;
        const float g = SPLIT ? ldg_split(gp, a.nsplit, a.split_stride) : __ldg(gp);
        const float u = __ldg(a.U + (long long)r * rs + nn);
        float sg;
        if (KIND == SURR_TRIANGLE) {
            sg = a.gamma * fmaxf(0.0f, 1.0f - fabsf(u - th) * inv_th);
        } else {
            const float dd = 1.0f + a.gamma * fabsf(u - th);
            sg = __frcp_rn(dd * dd);
        }
        return sg * g;
    };
    const int L = (a.R + NCH - 1) / NCH;
    const int lo = min(a.R, j * L), hi = min(a.R, lo + L);
    // 1. this chunk's map: delta_lo = A * delta_hi + Bv
    float A = 1.0f, Bv = 0.0f;
    if (act)
        for (int r = hi - 1; r >= lo; --r) {
            Bv = c_at(r) + lam * Bv;
            A *= lam;
        }
    // 2. compose the four maps of this neuron from the carry (after the last row) down to chunk 0
    float Ak[NCH], Bk[NCH];
#pragma unroll
    for (int k = 0; k < NCH; ++k) {
        Ak[k] = __shfl_sync(0xffffffffu, A, k * NPW + q);
        Bk[k] = __shfl_sync(0xffffffffu, Bv, k * NPW + q);
    }
    float din = act ? a.carry[nn] : 0.0f;   // delta after chunk NCH-1
    float mine = din;
#pragma unroll
    for (int k = NCH - 1; k >= 0; --k) {
        if (k == j) mine = din;             // delta after this lane's chunk
        din = Ak[k] * din + Bk[k];
    }
    // 3. re-walk the chunk from its incoming delta, emitting every delta_r
    float d = mine;
    if (act)
        for (int r = hi - 1; r >= lo; --r) {
            d = c_at(r) + lam * d;
            if (a.delta) a.delta[(long long)r * rs + n] = f2bf_bits(d);
        }
    if (act && j == 0) a.carry[n] = lo < hi ? d : mine;
}

cudaError_t launch_lif_bwd(const ScanBwdArgs &a, cudaStream_t s) {
    if (a.C % 4) return cudaErrorInvalidValue;
    const long long rs = (long long)a.B * a.H * a.W * a.C;
    if (rs == 0 || a.R == 0) return cudaSuccess;
    if (a.res_delta && (a.pool || a.H * a.W == 1 || a.res_lo % 4 || a.res_stride < 1 || a.H % a.res_stride ||
                        a.W % a.res_stride))
        return cudaErrorInvalidValue;
    if (!a.g_pooled && !a.res_delta && a.H * a.W == 1 && rs <= (1LL << 20)) {  // fc layers
        static const bool warp_off = getenv("SKIPPER_NO_WARP_SCAN") && atoi(getenv("SKIPPER_NO_WARP_SCAN"));
        if (a.R >= 16 && !warp_off) {   // long segments: the warp-parallel affine scan
            const unsigned grid = (unsigned)((rs + 63) / 64);   // 8 warps x 8 neurons per block
            const bool tri = a.surr == SURR_TRIANGLE;
            if (a.nsplit > 1) {
                if (tri) sk_launch(lif_bwd_warp_kernel<1, SURR_TRIANGLE>, grid, 256, 0, s, a);
                else sk_launch(lif_bwd_warp_kernel<1, SURR_FAST_SIGMOID>, grid, 256, 0, s, a);
            } else {
                if (tri) sk_launch(lif_bwd_warp_kernel<0, SURR_TRIANGLE>, grid, 256, 0, s, a);
                else sk_launch(lif_bwd_warp_kernel<0, SURR_FAST_SIGMOID>, grid, 256, 0, s, a);
            }
            return cudaGetLastError();
        }
        if (a.nsplit > 1)
            sk_launch(lif_bwd_small_kernel<SK_BS_CH_SPLIT, 1>, (unsigned)((rs + 255) / 256), 256, 0, s, a);
        else
            sk_launch(lif_bwd_small_kernel<16, 0>, (unsigned)((rs + 255) / 256), 256, 0, s, a);
        return cudaGetLastError();
    }
    const long long P = rs / 4;
    const unsigned grid = (unsigned)((P + 255) / 256);
    const bool tri = a.surr == SURR_TRIANGLE;
    // rows per unrolled chunk: 1 for short segments (per-segment SKIP schedules of a few kept rows: cfg 2 step
    // 5.867 -> 5.832 ms in alternating runs, the leaner loop co-resides better with the side-stream weight
    // gradients), 2 for long ones (cfg 4's 30-row segments measured 1 % slower with 1)
    const bool ch1 = a.R <= SK_BWD_CH1_MAX_R;
#define BWD_LAUNCH(SPL, KND)                                                         \
    do {                                                                             \
        if (ch1) sk_launch(lif_bwd_kernel<SPL, KND, 1>, grid, 256, 0, s, a);        \
        else sk_launch(lif_bwd_kernel<SPL, KND, SK_BWD_CH>, grid, 256, 0, s, a);   \
    } while (0)
    if (a.nsplit > 1) {
        if (tri) BWD_LAUNCH(1, SURR_TRIANGLE);
        else BWD_LAUNCH(1, SURR_FAST_SIGMOID);
    } else {
        if (tri) BWD_LAUNCH(0, SURR_TRIANGLE);
        else BWD_LAUNCH(0, SURR_FAST_SIGMOID);
    }
#undef BWD_LAUNCH
    return cudaGetLastError();
}

// Layer-0 operand rows for the timesteps of one segment (FIRST: t0 + r; RECOMPUTE: the kept list),
// straight from the uint8 input.  kind 0: bf16 copy of x[t] (fc or conv-with-wide-Cin input);
// kind 1: im2col of a 3x3 / pad-1 window, k = (dy*3+dx)*C0 + ci, zero-padded to K0 columns.
// SAM term l = 0 (Eq.4) is counted when s_part is given (FIRST pass only).
__global__ void stage_rows_kernel(const uint8_t *__restrict__ x, uint16_t *__restrict__ dst, const int *rows, int t0,
                                  int R, int B, int H, int W, int C0, int kind, int K0, long long D,
                                  unsigned *s_part, int stride) {
    pdl_enter();
    const long long per_row = kind == 1 ? (long long)B * H * W : (long long)B * D;
    const long long total = (long long)R * per_row;
    const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    long long t = -1;
    unsigned cnt = 0;
    if (i < total) {
        const int r = (int)(i / per_row);
        const long long e = i % per_row;
        t = rows ? rows[r] : t0 + r;
        if (kind == 1) {
            const int xx = (int)(e % W);
            const int yy = (int)((e / W) % H);
            const long long b = e / ((long long)H * W);
            const int Hi = H * stride, Wi = W * stride;  // input image (H x W output pixels)
            const uint8_t *xt = x + (t * B + b) * (long long)Hi * Wi * C0;
            uint64_t m = 0;  // bit k = im2col column k (registers only: no dynamically indexed arrays)
            for (int dy = 0; dy < 3; ++dy) {
                const int y = stride * yy + dy - 1;
                if (y < 0 || y >= Hi) continue;
                for (int dx = 0; dx < 3; ++dx) {
                    const int xq = stride * xx + dx - 1;
                    if (xq < 0 || xq >= Wi) continue;
                    const uint8_t *px = xt + ((long long)y * Wi + xq) * C0;
                    for (int ci = 0; ci < C0; ++ci)
                        if (__ldg(px + ci)) m |= 1ull << ((dy * 3 + dx) * C0 + ci);
                }
            }
            if (s_part)  // SAM l = 0: this output pixel's stride x stride block of input pixels
                for (int sy = 0; sy < stride; ++sy)
                    for (int sx = 0; sx < stride; ++sx) {
                        const uint8_t *pc = xt + ((long long)(stride * yy + sy) * Wi + stride * xx + sx) * C0;
                        for (int ci = 0; ci < C0; ++ci) cnt += __ldg(pc + ci) ? 1u : 0u;
                    }
            uint4 *o = reinterpret_cast<uint4 *>(dst + i * K0);
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                if (q < K0 / 8) {
                    uint32_t w[4];
#pragma unroll
                    for (int h = 0; h < 4; ++h) {
                        const int k = 8 * q + 2 * h;
                        w[h] = (((m >> k) & 1ull) ? 0x3F80u : 0u) | (((m >> (k + 1)) & 1ull) ? 0x3F800000u : 0u);
                    }
                    o[q] = make_uint4(w[0], w[1], w[2], w[3]);
                }
            }
        } else {
            const uint8_t v = x[t * (long long)B * D + e];
            dst[i] = v ? (uint16_t)0x3F80 : (uint16_t)0;
            cnt = v ? 1u : 0u;
        }
    }
    if (s_part) {
        const unsigned mask = 0xffffffffu;
        const long long tl = __shfl_sync(mask, t, 0);
        const bool same = __all_sync(mask, t == tl || t < 0);
        if (same) {
            const unsigned tot = __reduce_add_sync(mask, cnt);
            if ((threadIdx.x & 31) == 0 && tot && tl >= 0) atomicAdd(s_part + tl * 32 + (blockIdx.x & 31), tot);
        } else if (cnt) {
            atomicAdd(s_part + t * 32 + (blockIdx.x & 31), cnt);
        }
    }
}

cudaError_t launch_stage_rows(const uint8_t *x, uint16_t *dst, const int *rows, int t0, int R, int B, int H, int W,
                              int C0, int kind, int K0, long long D, unsigned *s_part, cudaStream_t s, int stride) {
    const long long per_row = kind == 1 ? (long long)B * H * W : (long long)B * D;
    const long long total = (long long)R * per_row;
    if (total == 0) return cudaSuccess;
    if (kind == 1 && (K0 % 8 || K0 > 64 || 9 * C0 > K0 || stride < 1 || stride > 2)) return cudaErrorInvalidValue;
    sk_launch(stage_rows_kernel, (unsigned)((total + 255) / 256), 256, 0, s, x, dst, rows, t0, R, B, H, W, C0, kind, K0, D,
                                                                     s_part, stride);
    return cudaGetLastError();
}

// ---------------------------------------------------------------------------- narrow / strided convs
// One thread per (output pixel, tap, 8-channel chunk): 16-byte load (or zero) -> 16-byte store.
// One thread per 16-byte chunk (8 channels) of a column row.  32-bit index math with the channel-chunk
// count as a template constant (the 64-bit div/mod chain of a generic version made this kernel
// integer-issue bound, 0.34 of HBM on cfg 4).
template <int C8>
__global__ void im2col_bf16_kernel(const uint16_t *__restrict__ X, uint16_t *__restrict__ cols, unsigned total,
                                   int Hin, int Win, int Cin, int H, int W, int stride) {
    pdl_enter();
    const unsigned i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= total) return;
    const int ch = (int)(i % C8);
    const unsigned q = i / C8;
    const int tap = (int)(q % 9u);
    const unsigned m = q / 9u;
    const unsigned my = m / (unsigned)W;
    const int x = (int)(m - my * (unsigned)W);
    const unsigned n = my / (unsigned)H;
    const int y = (int)(my - n * (unsigned)H);
    const int yi = stride * y + tap / 3 - 1, xi = stride * x + tap % 3 - 1;
    uint4 v = make_uint4(0u, 0u, 0u, 0u);
    if (yi >= 0 && yi < Hin && xi >= 0 && xi < Win)
        v = __ldg(reinterpret_cast<const uint4 *>(X + (((long long)n * Hin + yi) * Win + xi) * Cin) + ch);
    reinterpret_cast<uint4 *>(cols)[i] = v;
}

__global__ void im2col_bf16_kernel_l(const uint16_t *__restrict__ X, uint16_t *__restrict__ cols, long long total,
                                     int Hin, int Win, int Cin, int H, int W, int stride) {
    pdl_enter();
    const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= total) return;
    const int C8 = Cin >> 3;
    const int ch = (int)(i % C8);
    const long long q = i / C8;
    const int tap = (int)(q % 9);
    const long long m = q / 9;
    const int x = (int)(m % W), y = (int)((m / W) % H);
    const long long n = m / ((long long)H * W);
    const int yi = stride * y + tap / 3 - 1, xi = stride * x + tap % 3 - 1;
    uint4 v = make_uint4(0u, 0u, 0u, 0u);
    if (yi >= 0 && yi < Hin && xi >= 0 && xi < Win)
        v = __ldg(reinterpret_cast<const uint4 *>(X + ((n * Hin + yi) * Win + xi) * Cin) + ch);
    reinterpret_cast<uint4 *>(cols)[i] = v;
}

cudaError_t launch_im2col_bf16(const uint16_t *X, uint16_t *cols, long long nb, int Hin, int Win, int Cin, int H,
                               int W, int stride, cudaStream_t s) {
    if (Cin % 8) return cudaErrorInvalidValue;
    const long long total = nb * H * W * 9 * (Cin / 8);
    if (total == 0) return cudaSuccess;
    const unsigned blocks = (unsigned)((total + 255) / 256);
    if (total < (1LL << 31)) {
        const unsigned t = (unsigned)total;
        switch (Cin / 8) {
            case 2: sk_launch(im2col_bf16_kernel<2>, blocks, 256, 0, s, X, cols, t, Hin, Win, Cin, H, W, stride); return cudaGetLastError();
            case 4: sk_launch(im2col_bf16_kernel<4>, blocks, 256, 0, s, X, cols, t, Hin, Win, Cin, H, W, stride); return cudaGetLastError();
            case 8: sk_launch(im2col_bf16_kernel<8>, blocks, 256, 0, s, X, cols, t, Hin, Win, Cin, H, W, stride); return cudaGetLastError();
        }
    }
    sk_launch(im2col_bf16_kernel_l, blocks, 256, 0, s, X, cols, total, Hin, Win, Cin, H, W, stride);
    return cudaGetLastError();
}

// One thread per input neuron (n, yi, xi, ci): the <= 9 tap contributions in fixed order (deterministic).
template <typename IT>
__global__ void col2im_f32_kernel(const float *__restrict__ dcols, float *__restrict__ G, IT total, int Hin,
                                  int Win, int Cin, int H, int W, int stride) {
    pdl_enter();
    const IT i = (IT)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= total) return;
    const IT pix = i / (IT)Cin;
    const int ci = (int)(i - pix * (IT)Cin);
    const IT py = pix / (IT)Win;
    const int xi = (int)(pix - py * (IT)Win);
    const IT nn = py / (IT)Hin;
    const int yi = (int)(py - nn * (IT)Hin);
    const long long n = (long long)nn;
    float acc = 0.f;
#pragma unroll
    for (int dy = 0; dy < 3; ++dy) {
        const int ys = yi + 1 - dy;
        if (ys < 0 || ys % stride) continue;
        const int y = ys / stride;
        if (y >= H) continue;
#pragma unroll
        for (int dx = 0; dx < 3; ++dx) {
            const int xs = xi + 1 - dx;
            if (xs < 0 || xs % stride) continue;
            const int x = xs / stride;
            if (x >= W) continue;
            acc = __fadd_rn(acc, __ldg(dcols + ((n * H + y) * W + x) * 9LL * Cin + ci * 9 + dy * 3 + dx));
        }
    }
    G[i] = acc;
}

cudaError_t launch_col2im_f32(const float *dcols, float *G, long long nb, int Hin, int Win, int Cin, int H, int W,
                              int stride, cudaStream_t s) {
    const long long total = nb * Hin * Win * Cin;
    if (total == 0) return cudaSuccess;
    if (total < (1LL << 31))  // 32-bit index math (the 64-bit div/mod chain is integer-issue bound)
        sk_launch(col2im_f32_kernel<unsigned>, (unsigned)((total + 255) / 256), 256, 0, s, dcols, G, (unsigned)total, Hin,
                  Win, Cin, H, W, stride);
    else
        sk_launch(col2im_f32_kernel<long long>, (unsigned)((total + 255) / 256), 256, 0, s, dcols, G, total, Hin, Win, Cin,
                  H, W, stride);
    return cudaGetLastError();
}

// Global average pool (reading 23): one thread per (b, c), positions summed in order, then / P (exact for
// spike counts: integers < 2^24 and P a power of two in the supported networks).
__global__ void gap_reduce_kernel(const float *__restrict__ in, float *__restrict__ out, int B, int P, int C) {
    pdl_enter();
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= B * C) return;
    const int b = i / C, c = i % C;
    float acc = 0.f;
    for (int p = 0; p < P; ++p) acc += in[((long long)b * P + p) * C + c];
    out[i] = acc / (float)P;
}

__global__ void gap_expand_kernel(const float *__restrict__ g, float *__restrict__ out, int B, int P, int C) {
    pdl_enter();
    const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= (long long)B * P * C) return;
    const int c = (int)(i % C);
    const long long b = i / ((long long)P * C);
    out[i] = g[b * C + c] / (float)P;
}

cudaError_t launch_gap_reduce(const float *in, float *out, int B, int P, int C, cudaStream_t s) {
    sk_launch(gap_reduce_kernel, (B * C + 255) / 256, 256, 0, s, in, out, B, P, C);
    return cudaGetLastError();
}

cudaError_t launch_gap_expand(const float *g, float *out, int B, int P, int C, cudaStream_t s) {
    const long long n = (long long)B * P * C;
    sk_launch(gap_expand_kernel, (unsigned)((n + 255) / 256), 256, 0, s, g, out, B, P, C);
    return cudaGetLastError();
}

// dst[r][c] = bf16(src[r][c]) for c < cols, 0 for cols <= c < ld   (layer-0 weights padded to K0)
__global__ void cast_pad_bf16_kernel(const float *src, uint16_t *dst, int rows, int cols, int ld) {
    pdl_enter();
    const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= (long long)rows * ld) return;
    const int r = (int)(i / ld), c = (int)(i % ld);
    dst[i] = c < cols ? f2bf_bits(src[(long long)r * cols + c]) : (uint16_t)0;
}

cudaError_t launch_cast_pad_bf16(const float *src, uint16_t *dst, int rows, int cols, int ld, cudaStream_t s) {
    const long long n = (long long)rows * ld;
    sk_launch(cast_pad_bf16_kernel, (unsigned)((n + 255) / 256), 256, 0, s, src, dst, rows, cols, ld);
    return cudaGetLastError();
}

// dst[r][c] = src[r][c] for c < cols  (padded weight gradient back to [rows][cols])
__global__ void unpad_f32_kernel(const float *src, float *dst, int rows, int cols, int ld) {
    pdl_enter();
    const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= (long long)rows * cols) return;
    const int r = (int)(i / cols), c = (int)(i % cols);
    dst[i] = src[(long long)r * ld + c];
}

cudaError_t launch_unpad_f32(const float *src, float *dst, int rows, int cols, int ld, cudaStream_t s) {
    const long long n = (long long)rows * cols;
    sk_launch(unpad_f32_kernel, (unsigned)((n + 255) / 256), 256, 0, s, src, dst, rows, cols, ld);
    return cudaGetLastError();
}

__global__ void sam_finalize_kernel(const unsigned *s_part, long long *s, int T) {
    pdl_enter();
    const int t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= T) return;
    long long tot = 0;
    for (int i = 0; i < 32; ++i) tot += s_part[t * 32 + i];
    s[t] = tot;
}

// ---------------------------------------------------------------------------- Poisson encoder (NEXT-3)
// o0_t = [u_t < x * r_t].  u from Philox4x32-10 (counter = element index / 4, key = seed),
// u = (word >> 8) * 2^-24; x * r_t rounded once in fp32 - the oracle (oracle/encoder.py) draws the same.
SK_DEV void philox4x32_10(uint32_t c[4], uint32_t k0, uint32_t k1) {
#pragma unroll
    for (int r = 0; r < 10; ++r) {
        const uint32_t hi0 = __umulhi(0xD2511F53u, c[0]), lo0 = 0xD2511F53u * c[0];
        const uint32_t hi1 = __umulhi(0xCD9E8D57u, c[2]), lo1 = 0xCD9E8D57u * c[2];
        const uint32_t n0 = hi1 ^ c[1] ^ k0, n2 = hi0 ^ c[3] ^ k1;
        c[0] = n0;
        c[1] = lo1;
        c[2] = n2;
        c[3] = lo0;
        k0 += 0x9E3779B9u;
        k1 += 0xBB67AE85u;
    }
}

__global__ void poisson_encode_kernel(const float *__restrict__ x, const float *__restrict__ rates,
                                      unsigned long long seed, long long n, long long BD, uint8_t *__restrict__ out) {
    pdl_enter();
    const long long q = (long long)blockIdx.x * blockDim.x + threadIdx.x;  // one Philox block = 4 elements
    if (4 * q >= n) return;
    uint32_t c[4] = {(uint32_t)q, (uint32_t)((unsigned long long)q >> 32), 0u, 0u};
    philox4x32_10(c, (uint32_t)seed, (uint32_t)(seed >> 32));
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        const long long e = 4 * q + j;
        if (e >= n) break;
        const float u = (float)(c[j] >> 8) * 5.9604644775390625e-08f;  // 2^-24
        const float thr = __fmul_rn(__ldg(x + e % BD), __ldg(rates + e / BD));
        out[e] = u < thr ? 1 : 0;
    }
}

cudaError_t launch_poisson_encode(const float *x, const float *rates, unsigned long long seed, int T, int B, long long D,
                                  uint8_t *out, cudaStream_t s) {
    const long long n = (long long)T * B * D;
    const long long blocks = (n + 4 * 256 - 1) / (4 * 256);
    if (n == 0) return cudaSuccess;
    sk_launch(poisson_encode_kernel, (unsigned)blocks, 256, 0, s, x, rates, seed, n, (long long)B * D, out);
    return cudaGetLastError();
}

__global__ void sum32_f64_kernel(const double *part, double *out, int T) {
    pdl_enter();
    const int t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= T) return;
    double tot = 0.0;
    for (int i = 0; i < 32; ++i) tot += part[t * 32 + i];
    out[t] = tot;
}

cudaError_t launch_sum32_f64(const double *part, double *out, int T, cudaStream_t st) {
    sk_launch(sum32_f64_kernel, (T + 255) / 256, 256, 0, st, part, out, T);
    return cudaGetLastError();
}

cudaError_t launch_sam_finalize(const unsigned *s_part, long long *s, int T, cudaStream_t st) {
    sk_launch(sam_finalize_kernel, (T + 255) / 256, 256, 0, st, s_part, s, T);
    return cudaGetLastError();
}

// ============================================================================ readout + loss
// z[b][k] = (1/T) sum_n W^L[k][n] cnt[b][n]: one warp per (b, k)
__global__ void readout_z_kernel(const uint16_t *__restrict__ WbL, const float *__restrict__ cnt, float *z, int B, int D,
                                 int K, float invT) {
    pdl_enter();
    const long long w = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (w >= (long long)B * K) return;
    const int b = (int)(w / K), k = (int)(w % K);
    const uint16_t *wr = WbL + (long long)k * D;
    const float *cb = cnt + (long long)b * D;
    float acc = 0.f;
    for (int n = lane; n < D; n += 32) acc += bf_bits2f(wr[n]) * cb[n];
    for (int o = 16; o; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (lane == 0) z[w] = acc * invT;
}

// softmax cross-entropy, one block: warp w takes samples w, w + 8, ...; dz per sample, and loss += the
// per-sample CE / B_global summed in sample order by one thread (deterministic, no float atomics)
__global__ void readout_ce_kernel(const float *z, const int *labels, float *dz, float *loss, int B, int K, float invBg) {
    pdl_enter();
    extern __shared__ float s_ce[];  // [B]
    const int lane = threadIdx.x & 31;
    for (int b = threadIdx.x >> 5; b < B; b += blockDim.x >> 5) {
        const float *zb = z + (long long)b * K;
        float mx = -INFINITY;
        for (int k = lane; k < K; k += 32) mx = fmaxf(mx, zb[k]);
        for (int o = 16; o; o >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        float se = 0.f;
        for (int k = lane; k < K; k += 32) se += expf(zb[k] - mx);
        for (int o = 16; o; o >>= 1) se += __shfl_xor_sync(0xffffffffu, se, o);
        const int y = labels[b];
        for (int k = lane; k < K; k += 32) {
            const float pr = expf(zb[k] - mx) / se;
            dz[(long long)b * K + k] = (pr - (k == y ? 1.f : 0.f)) * invBg;
        }
        if (lane == 0) s_ce[b] = (logf(se) + mx - zb[y]) * invBg;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        float acc = 0.f;
        for (int b = 0; b < B; ++b) acc += s_ce[b];
        *loss += acc;
    }
}

// g_last[b][n] = (1/T) sum_k dz[b][k] W^L[k][n]: the gradient wrt the readout input, same at every t
__global__ void readout_g_kernel(const uint16_t *__restrict__ WbL, const float *__restrict__ dz, float *g_last, int B,
                                 int D, int K, float invT) {
    pdl_enter();
    const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= (long long)B * D) return;
    const int b = (int)(i / D), n = (int)(i % D);
    const float *db = dz + (long long)b * K;
    float acc = 0.f;
    for (int k = 0; k < K; ++k) acc += __ldg(db + k) * bf_bits2f(WbL[(long long)k * D + n]);
    g_last[i] = acc * invT;
}

cudaError_t launch_readout_loss(const uint16_t *WbL, const float *cnt, const int *labels, float *z, float *dz,
                                float *loss, float *g_last, int B, int D, int K, float invT, float invBg,
                                cudaStream_t s) {
    const long long warps = (long long)B * K;
    sk_launch(readout_z_kernel, (unsigned)((warps * 32 + 255) / 256), 256, 0, s, WbL, cnt, z, B, D, K, invT);
    if ((size_t)B * 4 > 48 * 1024) return cudaErrorInvalidValue;
    sk_launch(readout_ce_kernel, 1, 256, (size_t)B * 4, s, z, labels, dz, loss, B, K, invBg);
    const long long n = (long long)B * D;
    sk_launch(readout_g_kernel, (unsigned)((n + 255) / 256), 256, 0, s, WbL, dz, g_last, B, D, K, invT);
    return cudaGetLastError();
}

__global__ void readout_wgrad_kernel(const float *dz, const float *cnt_kept, float *dWL, int B, int D, int K, float invT,
                                     int accumulate) {
    pdl_enter();
    const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= (long long)K * D) return;
    const int k = (int)(i / D), n = (int)(i % D);
    float acc = 0.f;
#pragma unroll 16
    for (int b = 0; b < B; ++b) acc += dz[(long long)b * K + k] * cnt_kept[(long long)b * D + n];  // b ascending
    dWL[i] = accumulate ? dWL[i] + acc * invT : acc * invT;
}

cudaError_t launch_readout_wgrad(const float *dz, const float *cnt_kept, float *dWL, int B, int D, int K, float invT,
                                 cudaStream_t s, int accumulate) {
    const long long n = (long long)K * D;
    sk_launch(readout_wgrad_kernel, (unsigned)((n + 255) / 256), 256, 0, s, dz, cnt_kept, dWL, B, D, K, invT, accumulate);
    return cudaGetLastError();
}

// ============================================================================ split-K weight-gradient slices
// dst += sum of the nslices partial weight gradients (deterministic split-K, STORE_SLICE_ADD / narrow_wgrad),
// and the slices are zeroed for the next step.  A block owns 32 float4 columns; its 8 warps each sum a fixed
// contiguous range of the slices (independent loads, in slice order), and warp 0 adds the 8 partials in
// warp order - a fixed summation tree, so the result does not depend on scheduling.
__global__ void __launch_bounds__(256) reduce_slices_kernel(float4 *__restrict__ slices, int nslices,
                                                            float4 *__restrict__ dst, long long count4, int zero) {
    pdl_enter();
    __shared__ float4 part[8][32];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const long long i = (long long)blockIdx.x * 32 + lane;
    const int per = (nslices + 7) / 8, s0 = w * per, s1 = min(nslices, s0 + per);
    float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
    if (i < count4) {
        int s = s0;
        for (; s + 4 <= s1; s += 4) {  // four independent loads in flight, then the ordered adds
            float4 v[4];
#pragma unroll
            for (int k = 0; k < 4; ++k) v[k] = slices[(long long)(s + k) * count4 + i];
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                acc.x += v[k].x; acc.y += v[k].y; acc.z += v[k].z; acc.w += v[k].w;
                if (zero) slices[(long long)(s + k) * count4 + i] = make_float4(0.f, 0.f, 0.f, 0.f);
            }
        }
        for (; s < s1; ++s) {
            const float4 v = slices[(long long)s * count4 + i];
            acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
            if (zero) slices[(long long)s * count4 + i] = make_float4(0.f, 0.f, 0.f, 0.f);
        }
    }
    part[w][lane] = acc;
    __syncthreads();
    if (w == 0 && i < count4) {
        float4 t = part[0][lane];
#pragma unroll
        for (int k = 1; k < 8; ++k) {
            t.x += part[k][lane].x; t.y += part[k][lane].y; t.z += part[k][lane].z; t.w += part[k][lane].w;
        }
        float4 d = dst[i];
        d.x += t.x; d.y += t.y; d.z += t.z; d.w += t.w;
        dst[i] = d;
    }
}

cudaError_t launch_reduce_slices(float *slices, int nslices, float *dst, size_t count, cudaStream_t s, int zero) {
    if (count % 4 || (reinterpret_cast<uintptr_t>(slices) & 15) || (reinterpret_cast<uintptr_t>(dst) & 15))
        return cudaErrorInvalidValue;
    const long long c4 = (long long)(count / 4);
    if (c4 == 0 || nslices <= 0) return cudaSuccess;
    sk_launch(reduce_slices_kernel, (unsigned)((c4 + 31) / 32), 256, 0, s, reinterpret_cast<float4 *>(slices), nslices,
              reinterpret_cast<float4 *>(dst), c4, zero);
    return cudaGetLastError();
}

// ============================================================================ Adam + shadows
template <int VEC>
__global__ void adam_kernel(float *w, const float *g, float *m, float *v, uint16_t *wb, long long n, float lr, float b1,
                            float b2, float eps, float bc1, float bc2_sqrt) {
    pdl_enter();
    // VEC: 4 parameters per thread (16-byte loads / stores); the per-element arithmetic is the same
    const long long i4 = ((long long)blockIdx.x * blockDim.x + threadIdx.x) * (VEC ? 4 : 1);
    if (i4 >= n) return;
    auto upd = [&](float wi, float gi, float &mi, float &vi) {
        mi = b1 * mi + (1.f - b1) * gi;
        vi = b2 * vi + (1.f - b2) * gi * gi;
        return wi - (lr / bc1) * mi / (sqrtf(vi) / bc2_sqrt + eps);
    };
    if (VEC && i4 + 4 <= n) {
        float4 w4 = *reinterpret_cast<const float4 *>(w + i4);
        const float4 g4 = *reinterpret_cast<const float4 *>(g + i4);
        float4 m4 = *reinterpret_cast<const float4 *>(m + i4);
        float4 v4 = *reinterpret_cast<const float4 *>(v + i4);
        w4.x = upd(w4.x, g4.x, m4.x, v4.x);
        w4.y = upd(w4.y, g4.y, m4.y, v4.y);
        w4.z = upd(w4.z, g4.z, m4.z, v4.z);
        w4.w = upd(w4.w, g4.w, m4.w, v4.w);
        *reinterpret_cast<float4 *>(m + i4) = m4;
        *reinterpret_cast<float4 *>(v + i4) = v4;
        *reinterpret_cast<float4 *>(w + i4) = w4;
        *reinterpret_cast<uint2 *>(wb + i4) = make_uint2(f2bf_bits(w4.x) | ((uint32_t)f2bf_bits(w4.y) << 16),
                                                         f2bf_bits(w4.z) | ((uint32_t)f2bf_bits(w4.w) << 16));
    } else {
        for (long long i = i4; i < n && i < i4 + (VEC ? 4 : 1); ++i) {
            float mi = m[i], vi = v[i];
            const float wi = upd(w[i], g[i], mi, vi);
            m[i] = mi;
            v[i] = vi;
            w[i] = wi;
            wb[i] = f2bf_bits(wi);
        }
    }
}

cudaError_t launch_adam(float *w, const float *g, float *m, float *v, uint16_t *wb, size_t n, float lr, float b1,
                        float b2, float eps, float bc1, float bc2_sqrt, cudaStream_t s) {
    if (n == 0) return cudaSuccess;
    const bool aligned = ((reinterpret_cast<uintptr_t>(w) | reinterpret_cast<uintptr_t>(g) | reinterpret_cast<uintptr_t>(m) |
                           reinterpret_cast<uintptr_t>(v)) & 15) == 0 && (reinterpret_cast<uintptr_t>(wb) & 7) == 0;
    if (aligned) {
        const long long t = ((long long)n + 3) / 4;
        sk_launch(adam_kernel<1>, (unsigned)((t + 255) / 256), 256, 0, s, w, g, m, v, wb, (long long)n, lr, b1, b2, eps, bc1,
                  bc2_sqrt);
    } else {  // a layer's slice of the flat gradient buffer need not be 16-byte aligned
        sk_launch(adam_kernel<0>, (unsigned)((n + 255) / 256), 256, 0, s, w, g, m, v, wb, (long long)n, lr, b1, b2, eps, bc1,
                  bc2_sqrt);
    }
    return cudaGetLastError();
}

__global__ void cast_bf16_kernel(const float *w, uint16_t *wb, long long n) {
    pdl_enter();
    const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) wb[i] = f2bf_bits(w[i]);
}

cudaError_t launch_cast_bf16(const float *w, uint16_t *wb, size_t n, cudaStream_t s) {
    if (n == 0) return cudaSuccess;
    sk_launch(cast_bf16_kernel, (unsigned)((n + 255) / 256), 256, 0, s, w, wb, (long long)n);
    return cudaGetLastError();
}

// dst[c][t][a] = src[a][t][c]
__global__ void transpose_bf16_kernel(const uint16_t *src, uint16_t *dst, int A, int Tp, int Cc) {
    pdl_enter();
    __shared__ uint16_t tile[32][33];
    const int t = blockIdx.z;
    const int a0 = blockIdx.y * 32, c0 = blockIdx.x * 32;
    for (int i = threadIdx.y; i < 32; i += blockDim.y) {
        const int a = a0 + i, c = c0 + threadIdx.x;
        if (a < A && c < Cc) tile[i][threadIdx.x] = src[((long long)a * Tp + t) * Cc + c];
    }
    __syncthreads();
    for (int i = threadIdx.y; i < 32; i += blockDim.y) {
        const int c = c0 + i, a = a0 + threadIdx.x;
        if (a < A && c < Cc) dst[((long long)c * Tp + t) * A + a] = tile[threadIdx.x][i];
    }
}

cudaError_t launch_transpose_bf16(const uint16_t *src, uint16_t *dst, int A, int Tp, int Cc, cudaStream_t s) {
    dim3 grid((Cc + 31) / 32, (A + 31) / 32, Tp);
    sk_launch(transpose_bf16_kernel, grid, dim3(32, 8), 0, s, src, dst, A, Tp, Cc);
    return cudaGetLastError();
}

}  // namespace sk
