// conv_narrow.cu - 3x3 / pad-1 convolutions of narrow-channel (16..64) images on tcgen05, for the ResNet
// SNN layers (reading 8): forward with stride 1 or 2, and the stride-1 dgrad (flipped taps).
//
// A TMA box of a 16-channel image has 32-byte rows, and the TMA unit is row-issue bound on them
// (tools/conv_s_bench.py).  Here the activation tile of each tap is instead gathered by
// 128 producer threads with 16-byte cp.async (.ca: the 9 taps re-read the same pixels through L1),
// written in the no-swizzle K-major UMMA layout (one 2 KB plane per 8 channels: 128 pixel rows x 16 B,
// 8-row core matrices 128 B apart, planes LBO apart), so a pixel shift is just a different source address.
// The weights of all 9 taps stay resident in shared memory for the kernel's lifetime.
//
//   warps 0-3   producers: thread p gathers tile row p (one output pixel) for every tap
//   warp 4      TMEM allocator + MMA issuer (tcgen05.mma M=128, N=Cout, K=16 per instruction)
//   warps 5-8   epilogue: tcgen05.ld 32x32b -> fp32 rows of the output (one pixel row per thread)
//
// Y[n, y, x, co] = sum_{tap, ci} Wk[co][tap][ci] X[n, s*y + dy - 1, s*x + dx - 1, ci]  (sign = +1)
// G[n, y, x, ci] = sum_{tap, co} Wt[ci][tap][co] D[n, y - dy + 1, x - dx + 1, co]      (sign = -1, s = 1)
#include <algorithm>
#include <cstdio>
#include <cstdlib>

#include "common.cuh"
#include "gemm.h"

namespace sk {

static constexpr int CN_PROD = 128;       // producer threads (one per tile row)
static constexpr int CN_MMA_WARP = 4;
static constexpr int CN_EPI_WARP0 = 5;
static constexpr int CN_THREADS = 32 * (CN_EPI_WARP0 + 4);
static constexpr int CN_MAX_RING = 16;

SK_DEV void cp_async16(uint32_t dst, const void *src, uint32_t src_bytes) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src), "r"(src_bytes) : "memory");
}
template <int N>
SK_DEV void cp_async_wait_n() {  // at most N groups still pending
    asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}

// K-major, no swizzle: 8-row core matrices of 16 B rows, SBO = 128 B along M/N, LBO between 8-col K chunks
SK_DEV uint64_t cn_desc(uint32_t saddr, uint32_t lbo_bytes) {
    uint64_t d = 0;
    d |= (uint64_t)((saddr >> 4) & 0x3FFF);
    d |= (uint64_t)((lbo_bytes >> 4) & 0x3FFF) << 16;
    d |= (uint64_t)(128u >> 4) << 32;
    d |= (uint64_t)1 << 46;
    return d;
}

SK_DEV float cn_lif(float U, float I, float o, float lam, float th) {  // Eq.1, no FMA (oracle order)
    return __fsub_rn(__fadd_rn(__fmul_rn(lam, U), I), o != 0.f ? th : 0.f);  // theta * o, o in {0, 1}: exact select
}

// LIF = false: one conv over nb images (R = 1), fp32 output.  LIF = true: the tile is 128 pixels of one
// timestep row; the CTA walks the segment's rows for it, and the epilogue runs Eq.1 with the membranes of
// its pixel held in registers across the rows (conv_lif.cu's scheme for narrow layers).
template <int N, bool LIF>  // output channels (16..128, multiple of 16; LIF: 16 or 32)
__global__ void __launch_bounds__(CN_THREADS, LIF ? (N <= 16 ? 4 : 2) : 1) conv_narrow_kernel(const NarrowConvArgs a) {
    pdl_enter();
    constexpr int NACC = LIF ? 4 : 2;  // TMEM accumulator ring (the LIF epilogue is the slower consumer)
    constexpr uint32_t TMEM_COLS = (NACC * N <= 32) ? 32 : (NACC * N <= 64 ? 64 : (NACC * N <= 128 ? 128 : 256));
    extern __shared__ uint8_t smem_raw[];
    const uint32_t raw = smem_u32(smem_raw);
    const uint32_t base = (raw + 1023u) & ~1023u;
    const int KP = a.Cin / 8;                                 // 16-byte K planes per tap
    const uint32_t plane_a = 128u * 16u;                      // one plane of the A tile
    const uint32_t stage_bytes = (uint32_t)KP * plane_a;
    const uint32_t plane_b = (uint32_t)N * 16u;
    const uint32_t sB = base;                                 // [9][KP][N][16 B] resident weights
    const uint32_t b_bytes = 9u * KP * plane_b;
    const uint32_t sA = (sB + b_bytes + 1023u) & ~1023u;      // ring of A stages
    const int ring = a.ring;
    const uint32_t bars = sA + (uint32_t)ring * stage_bytes;
    auto full_bar = [&](int s) { return bars + 8u * s; };
    auto empty_bar = [&](int s) { return bars + 8u * (CN_MAX_RING + s); };
    auto tfull_bar = [&](int i) { return bars + 8u * (2 * CN_MAX_RING + i); };
    auto tempty_bar = [&](int i) { return bars + 8u * (2 * CN_MAX_RING + 4 + i); };
    const uint32_t tmem_slot = bars + 8u * (2 * CN_MAX_RING + 8);

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const long long HW = (long long)a.H * a.W;
    const long long M = (long long)a.nb * HW;                 // output pixels per row
    const int tiles = (int)((M + 127) / 128);
    const int R = LIF ? a.R : 1;
    const int r_mma0 = (LIF && a.restore) ? 1 : 0;            // RECOMPUTE: row 0 is the checkpoint
    const long long in_row = (long long)a.nb * a.Hin * a.Win * a.Cin;

    // resident weights: chunk (co, tap, k8) of Wk[co][tap][Cin] -> sB + (tap*KP + k8)*plane_b + co*16
    {
        const int chunks = N * 9 * KP;
        for (int e = threadIdx.x; e < chunks; e += blockDim.x) {
            const int k8 = e % KP, tap = (e / KP) % 9, co = e / (9 * KP);
            const uint4 v = *reinterpret_cast<const uint4 *>(a.Wk + ((long long)co * 9 + tap) * a.Cin + 8 * k8);
            *reinterpret_cast<uint4 *>(smem_raw + (sB - raw) + ((uint32_t)tap * KP + k8) * plane_b + (uint32_t)co * 16u) = v;
        }
    }
    fence_async_shared();
    if (threadIdx.x == 0) {
        for (int s = 0; s < ring; ++s) {
            mbar_init(full_bar(s), CN_PROD / 32);  // one arrival per producer warp
            mbar_init(empty_bar(s), 1);
        }
        for (int i = 0; i < NACC; ++i) {
            mbar_init(tfull_bar(i), 1);
            mbar_init(tempty_bar(i), 4);
        }
        fence_mbar_init();
    }
    if (warp == CN_MMA_WARP) tmem_alloc<TMEM_COLS>(tmem_slot);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *reinterpret_cast<volatile uint32_t *>(smem_raw + (tmem_slot - raw));

    if (warp < 4) {
        // ------------------------------------------------------------ producers
        const int p = threadIdx.x;  // tile row
        int stage = 0, issued = 0, signalled = 0;
        const int lag = ring >= 10 ? 8 : (ring >= 6 ? 4 : 2);  // stages in flight per thread (wait_group immediates)
        uint32_t phase = 0;
        int sig_stage = 0;
        for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
            const long long m = (long long)tile * 128 + p;
            const bool valid = m < M;
            const long long n = valid ? m / HW : 0;
            const int y = valid ? (int)((m / a.W) % a.H) : 0, x = valid ? (int)(m % a.W) : 0;
            for (int r = r_mma0; r < R; ++r) {
                const uint16_t *Xr = a.X + (long long)r * in_row;
                for (int tap = 0; tap < 9; ++tap) {
                    mbar_wait(empty_bar(stage), phase ^ 1u);
                    const int dy = tap / 3 - 1, dx = tap % 3 - 1;
                    const int yi = a.sign > 0 ? a.stride * y + dy : y - dy;
                    const int xi = a.sign > 0 ? a.stride * x + dx : x - dx;
                    const bool in = valid && yi >= 0 && yi < a.Hin && xi >= 0 && xi < a.Win;
                    const uint16_t *src = in ? Xr + ((n * a.Hin + yi) * a.Win + xi) * a.Cin : a.X;
                    const uint32_t dst = sA + (uint32_t)stage * stage_bytes + (uint32_t)p * 16u;
                    for (int j = 0; j < KP; ++j) cp_async16(dst + (uint32_t)j * plane_a, src + 8 * j, in ? 16u : 0u);
                    cp_async_commit();
                    ++issued;
                    if (++stage == ring) {
                        stage = 0;
                        phase ^= 1u;
                    }
                    if (issued - signalled > lag) {  // the oldest pending stage has landed: publish it
                        if (lag >= 8) cp_async_wait_n<8>();
                        else if (lag >= 4) cp_async_wait_n<4>();
                        else cp_async_wait_n<2>();
                        fence_async_shared();
                        __syncwarp();
                        if (lane == 0) mbar_arrive(full_bar(sig_stage));
                        ++signalled;
                        if (++sig_stage == ring) sig_stage = 0;
                    }
                }
            }
        }
        cp_async_wait_n<0>();
        fence_async_shared();
        __syncwarp();
        while (signalled < issued) {
            if (lane == 0) mbar_arrive(full_bar(sig_stage));
            ++signalled;
            if (++sig_stage == ring) sig_stage = 0;
        }
    } else if (warp == CN_MMA_WARP) {
        if (lane == 0) {
            // ------------------------------------------------------------ MMA issuer
            constexpr uint32_t idesc = umma_idesc_bf16(128, N, 0, 0);
            int stage = 0, acc = 0;
            uint32_t phase = 0, acc_phase = 0;
            for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
                for (int r = r_mma0; r < R; ++r) {
                    mbar_wait(tempty_bar(acc), acc_phase ^ 1u);
                    tc_fence_after();
                    const uint32_t d_tmem = tmem_base + (uint32_t)acc * N;
                    for (int tap = 0; tap < 9; ++tap) {
                        mbar_wait(full_bar(stage), phase);
                        tc_fence_after();
                        const uint32_t sa = sA + (uint32_t)stage * stage_bytes;
                        const uint32_t sb = sB + (uint32_t)tap * KP * plane_b;
                        for (int k = 0; k < KP / 2; ++k) {  // K = 16 per instruction = two 8-channel planes
                            const uint64_t ad = cn_desc(sa + (uint32_t)k * 2u * plane_a, plane_a);
                            const uint64_t bd = cn_desc(sb + (uint32_t)k * 2u * plane_b, plane_b);
                            tc_mma_f16(d_tmem, ad, bd, idesc, (tap > 0 || k > 0) ? 1u : 0u);
                        }
                        tc_commit(empty_bar(stage));
                        if (++stage == ring) {
                            stage = 0;
                            phase ^= 1u;
                        }
                    }
                    tc_commit(tfull_bar(acc));
                    if (++acc == NACC) {
                        acc = 0;
                        acc_phase ^= 1u;
                    }
                }
            }
        }
    } else if (!LIF) {
        // ---------------------------------------------------------------- epilogue (fp32 output)
        const int q = warp & 3;  // TMEM lane quadrant (warps 5, 6, 7, 8 -> 1, 2, 3, 0)
        int acc = 0;
        uint32_t acc_phase = 0;
        for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
            mbar_wait(tfull_bar(acc), acc_phase);
            tc_fence_after();
            const long long m = (long long)tile * 128 + q * 32 + lane;
            const bool valid = m < M;
            float *dst = a.Y + (valid ? m : 0) * (long long)a.Cout;
#pragma unroll
            for (int c = 0; c < N / 16; ++c) {
                uint32_t r[16];
                tmem_ld_32x32b_x16(tmem_base + ((uint32_t)(q * 32) << 16) + (uint32_t)acc * N + c * 16, r);
                tmem_ld_wait();
                if (valid) {
#pragma unroll
                    for (int i = 0; i < 16; i += 4)
                        *reinterpret_cast<float4 *>(dst + 16 * c + i) =
                            make_float4(__uint_as_float(r[i]), __uint_as_float(r[i + 1]), __uint_as_float(r[i + 2]),
                                        __uint_as_float(r[i + 3]));
                }
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(tempty_bar(acc));
            if (++acc == NACC) {
                acc = 0;
                acc_phase ^= 1u;
            }
        }
    } else {
        // ---------------------------------------------------------------- epilogue (Eq.1 over the rows)
        constexpr int NW = (N + 31) / 32;
        const int q = warp & 3;
        const long long rs = M * N;  // neurons per row
        int acc = 0;
        uint32_t acc_phase = 0;
        for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
            const long long m = (long long)tile * 128 + q * 32 + lane;
            const bool valid = m < M;
            const long long nidx = (valid ? m : 0) * N;
            float U[N];
            uint32_t ob[NW];
#pragma unroll
            for (int j = 0; j < NW; ++j) ob[j] = 0u;
            if (valid) {
#pragma unroll
                for (int c = 0; c < N; c += 4) {
                    const float4 u = *reinterpret_cast<const float4 *>(a.U_state + nidx + c);
                    U[c] = u.x; U[c + 1] = u.y; U[c + 2] = u.z; U[c + 3] = u.w;
                    const uchar4 o4 = *reinterpret_cast<const uchar4 *>(a.o_state + nidx + c);
                    ob[c >> 5] |= ((o4.x ? 1u : 0u) | (o4.y ? 2u : 0u) | (o4.z ? 4u : 0u) | (o4.w ? 8u : 0u)) << (c & 31);
                }
            } else {
#pragma unroll
                for (int c = 0; c < N; ++c) U[c] = 0.f;
            }
            // residual source offset of this pixel (reading 8): channels [res_lo, res_lo + res_C)
            long long roff = -1, rrs = 0;
            if (a.res && valid) {
                const long long n = m / HW;
                const int y = (int)((m / a.W) % a.H), x = (int)(m % a.W);
                rrs = (long long)a.nb * a.res_H * a.res_W * a.res_C;
                roff = ((n * a.res_H + (long long)y * a.res_stride) * a.res_W + (long long)x * a.res_stride) * a.res_C;
            }
            auto bitf = [&](int c) { return (float)((ob[c >> 5] >> (c & 31)) & 1u); };
            auto store_state = [&](float *Ud, uint8_t *od) {
#pragma unroll
                for (int c = 0; c < N; c += 4) {
                    *reinterpret_cast<float4 *>(Ud + c) = make_float4(U[c], U[c + 1], U[c + 2], U[c + 3]);
                    const uint32_t w = ob[c >> 5] >> (c & 31);
                    *reinterpret_cast<uchar4 *>(od + c) = make_uchar4(w & 1u, (w >> 1) & 1u, (w >> 2) & 1u, (w >> 3) & 1u);
                }
            };
            auto emit = [&](int r, bool counted) {
                const long long t = a.row_t ? (long long)a.row_t[r] : (long long)a.t0 + r;
                unsigned cnt = 0;
                double q2 = 0.0;
                if (valid) {
#pragma unroll
                    for (int j = 0; j < NW; ++j) cnt += __popc(ob[j]);
                    uint16_t *po = a.Po_out + (long long)r * rs + nidx;
#pragma unroll
                    for (int c = 0; c < N; c += 16) {  // 16 bf16 spikes = one 32-byte sector per store
                        const uint32_t w = ob[c >> 5] >> (c & 31);
                        uint32_t pk[8];
#pragma unroll
                        for (int e = 0; e < 8; ++e)
                            pk[e] = (((w >> (2 * e)) & 1u) ? 0x3F80u : 0u) | (((w >> (2 * e + 1)) & 1u) ? 0x3F800000u : 0u);
                        st_global_v8u(po + c, make_uint4(pk[0], pk[1], pk[2], pk[3]), make_uint4(pk[4], pk[5], pk[6], pk[7]));
                    }
                    if (a.U_out) {
                        float *du = a.U_out + (long long)r * rs + nidx;
#pragma unroll
                        for (int c = 0; c < N; c += 8) st_global_v8(du + c, U + c);
                    }
                    if (a.dbg_U) store_state(a.dbg_U + t * rs + nidx, a.dbg_o + t * rs + nidx);
                    if (a.cnt) {  // readout input sum (last spiking layer): this thread owns these neurons
#pragma unroll
                        for (int c = 0; c < N; c += 4) {
                            float4 *cp = reinterpret_cast<float4 *>(a.cnt + nidx + c);
                            float4 v = *cp;
                            v.x += bitf(c); v.y += bitf(c + 1); v.z += bitf(c + 2); v.w += bitf(c + 3);
                            *cp = v;
                        }
                    }
                    if (a.u2_part) {
#pragma unroll
                        for (int c = 0; c < N; ++c) q2 += (double)U[c] * (double)U[c];
                    }
                }
                if (counted && a.s_part) {
                    const unsigned v = __reduce_add_sync(0xffffffffu, cnt);
                    if (lane == 0 && v) atomicAdd(a.s_part + t * 32 + (blockIdx.x & 31), v);
                }
                if (counted && a.u2_part) u2_warp_add(a.u2_part, t, q2);
            };
            if (a.restore) emit(0, false);
            for (int r = r_mma0; r < R; ++r) {
                mbar_wait(tfull_bar(acc), acc_phase);
                tc_fence_after();
                float I[N];
#pragma unroll
                for (int c = 0; c < N / 16; ++c) {
                    uint32_t rr[16];
                    tmem_ld_32x32b_x16(tmem_base + ((uint32_t)(q * 32) << 16) + (uint32_t)acc * N + c * 16, rr);
                    tmem_ld_wait();
#pragma unroll
                    for (int i = 0; i < 16; ++i) I[16 * c + i] = __uint_as_float(rr[i]);
                }
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(tempty_bar(acc));
                if (++acc == NACC) {
                    acc = 0;
                    acc_phase ^= 1u;
                }
                if (roff >= 0) {  // I += S(a^r): exact (spikes added to the fp32 sum)
                    const uint16_t *rp = a.res + (long long)r * rrs + roff;
// 8 channels (16 bytes) per load: res_lo and res_C are multiples of 8 (launch check), so a chunk is
                    // wholly in or out
auto add8 = [&](int c8, const uint4 &v) {
                        const uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
                        for (int e = 0; e < 4; ++e) {
                            I[c8 + 2 * e] = __fadd_rn(I[c8 + 2 * e], __uint_as_float(w[e] << 16));
                            I[c8 + 2 * e + 1] = __fadd_rn(I[c8 + 2 * e + 1], __uint_as_float(w[e] & 0xffff0000u));
                        }
                    };
                    if (a.res_lo == 0 && a.res_C == N && N % 16 == 0) {  // identity shortcut: 32-byte loads (whole sectors)
#pragma unroll
                        for (int c16 = 0; c16 < N; c16 += 16) {
                            uint4 v0, v1;
                            ldg_v8u(rp + c16, v0, v1);
                            add8(c16, v0);
                            add8(c16 + 8, v1);
                        }
                    } else {
#pragma unroll
                        for (int c8 = 0; c8 < N; c8 += 8) {
                            const int cs = c8 - a.res_lo;
                            if (cs >= 0 && cs < a.res_C) add8(c8, __ldg(reinterpret_cast<const uint4 *>(rp + cs)));
                        }
                    }
                }
                uint32_t nb[NW];
#pragma unroll
                for (int j = 0; j < NW; ++j) nb[j] = 0u;
#pragma unroll
                for (int c = 0; c < N; ++c) {
                    U[c] = cn_lif(U[c], I[c], bitf(c), a.lam, a.theta);
                    nb[c >> 5] |= (U[c] > a.theta ? 1u : 0u) << (c & 31);
                }
#pragma unroll
                for (int j = 0; j < NW; ++j) ob[j] = nb[j];
                emit(r, true);
                if (a.ckU && (a.ck_every ? r % a.ck_every == 0 : r == 0) && valid) {
                    const long long slot = a.ck_every ? (long long)(r / a.ck_every) * a.ck_stride : 0;
                    store_state(a.ckU + slot + nidx, a.cko + slot + nidx);
                }
            }
            if (valid && !a.restore) store_state(a.U_state + nidx, a.o_state + nidx);
        }
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    if (warp == CN_MMA_WARP) tmem_dealloc<TMEM_COLS>(tmem_base);
}

bool conv_narrow_supported(int cin, int cout, int stride, int sign) {
    if (cin % 16 || cin < 16 || cin > 64) return false;
    if (cout % 16 || cout < 16 || cout > 128) return false;
    if (stride != 1 && stride != 2) return false;
    if (sign == -1 && stride != 1) return false;
    return true;
}

template <int N, bool LIF>
static cudaError_t launch_n(NarrowConvArgs a, cudaStream_t s, int num_sms) {
    const int KP = a.Cin / 8;
    const uint32_t stage_bytes = (uint32_t)KP * 2048u;
    const uint32_t b_bytes = ((9u * KP * N * 16u) + 1023u) & ~1023u;
    // a 48 KB ring leaves room for several CTAs per SM: the gather is latency bound, so more resident
    // producer warps (not a deeper ring per CTA) is what feeds it
    static const int lif16_ctas = getenv("SKIPPER_NARROW_LIF_CTAS") ? atoi(getenv("SKIPPER_NARROW_LIF_CTAS")) : 4;
    const int want = LIF ? (N <= 16 ? lif16_ctas : 2) : 4;  // resident CTAs per SM aimed for
    a.ring = (int)std::max<uint32_t>(4u, std::min<uint32_t>(CN_MAX_RING, ((want >= 4 ? 48u : 64u) * 1024u) / stage_bytes));
    const size_t smem = 1024 + b_bytes + (size_t)a.ring * stage_bytes + 8 * (2 * CN_MAX_RING + 8) + 16;
    static bool attr = false;
    if (!attr) {
        cudaError_t e = cudaFuncSetAttribute(conv_narrow_kernel<N, LIF>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             227 * 1024);
        if (e != cudaSuccess) return e;
        attr = true;
    }
    // resident CTAs per SM from shared memory (228 KB per SM, 1 KB reserved per CTA) and registers; the
    // occupancy API reports 1 here (launch bounds), so computed
    // (the 16-channel LIF variant fits 56 registers without spills: 4 resident CTAs with a 48 KB ring)
    int per_sm = (int)std::min<size_t>(want, (228u * 1024u) / (smem + 1024));
    if (per_sm < 1) per_sm = 1;
    constexpr int nacc = LIF ? 4 : 2;
    constexpr int tmem_cols = (nacc * N <= 32) ? 32 : (nacc * N <= 64 ? 64 : (nacc * N <= 128 ? 128 : 256));
    per_sm = std::min(per_sm, 512 / tmem_cols);  // every resident CTA holds its TMEM accumulators
    const long long M = (long long)a.nb * a.H * a.W;
    const int tiles = (int)((M + 127) / 128);
    const int grid = (int)std::min<long long>(tiles, (long long)num_sms * per_sm);
    if (getenv("SKIPPER_NARROW_DEBUG"))
        fprintf(stderr, "[conv_narrow%s] N=%d cin=%d ring=%d smem=%zu per_sm=%d grid=%d tiles=%d\n", LIF ? "_lif" : "",
                N, a.Cin, a.ring, smem, per_sm, grid, tiles);
    if (grid <= 0) return cudaSuccess;
    sk_launch(conv_narrow_kernel<N, LIF>, grid, CN_THREADS, smem, s, a);
    return cudaGetLastError();
}

cudaError_t launch_conv_narrow(const NarrowConvArgs &a, cudaStream_t s, int num_sms) {
    if (!conv_narrow_supported(a.Cin, a.Cout, a.stride, a.sign)) return cudaErrorInvalidValue;
    switch (a.Cout) {
        case 16: return launch_n<16, false>(a, s, num_sms);
        case 32: return launch_n<32, false>(a, s, num_sms);
        case 48: return launch_n<48, false>(a, s, num_sms);
        case 64: return launch_n<64, false>(a, s, num_sms);
        case 96: return launch_n<96, false>(a, s, num_sms);
        case 128: return launch_n<128, false>(a, s, num_sms);
    }
    return cudaErrorInvalidValue;
}

bool conv_narrow_lif_supported(int cin, int cout, int stride) {
    return conv_narrow_supported(cin, cout, stride, 1) && (cout == 16 || cout == 32);
}

cudaError_t launch_conv_narrow_lif(const NarrowConvArgs &a0, cudaStream_t s, int num_sms) {
    NarrowConvArgs a = a0;
    a.sign = 1;
    if (!conv_narrow_lif_supported(a.Cin, a.Cout, a.stride) || a.R <= 0) return cudaErrorInvalidValue;
    if (a.res && (a.res_C % 8 || a.res_lo % 8 || a.res_lo < 0 || a.res_lo + a.res_C > a.Cout)) return cudaErrorInvalidValue;
    switch (a.Cout) {
        case 16: return launch_n<16, true>(a, s, num_sms);
        case 32: return launch_n<32, true>(a, s, num_sms);
    }
    return cudaErrorInvalidValue;
}

}  // namespace sk
