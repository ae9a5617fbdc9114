// narrow_lif.cu - fused 3x3 conv + LIF scan (Eq.1) for the 16-channel ResNet-DVS layers (cfg 4),
// on warp-level bf16 tensor-core MMAs instead of conv_narrow.cu's per-tap cp.async im2col + tcgen05.
//
// Work unit = 128 output pixels (whole image rows of one image) of every row (timestep) of the segment.
// Per row the CTA stages the input rows the band reads (one halo row above and below; stride 1 or 2) with
// cp.async, double-buffered so row r+1 streams in while row r is computed; 8 warps each compute 16 pixels
// x COUT channels of the synaptic current with mma.sync.m16n8k16 whose A rows (one per pixel and tap, or a
// zero row for the padding) are gathered by ldmatrix straight from the staged rows, B = the resident
// weights.  The fp32 currents go through a shared-memory tile to 128 epilogue threads (thread = pixel, all
// COUT channels, membranes in registers across the rows) that run exactly conv_narrow.cu's Eq.1 epilogue:
// residual shortcut, spikes, stored U, checkpoint, SAM counts, l2 trace, readout counts, debug record.
#include "common.cuh"
#include "gemm.h"

#include <algorithm>
#include <cstdio>
#include <cstdlib>

namespace sk {

namespace {
constexpr int NL_THREADS = 256;
constexpr int NL_P = 128;

SK_DEV void nl_ldsm_x4(uint32_t addr, uint32_t &r0, uint32_t &r1, uint32_t &r2, uint32_t &r3) {
    asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0, %1, %2, %3}, [%4];"
                 : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3)
                 : "r"(addr));
}
SK_DEV void nl_ldsm_x2(uint32_t addr, uint32_t &r0, uint32_t &r1) {
    asm volatile("ldmatrix.sync.aligned.m8n8.x2.shared.b16 {%0, %1}, [%2];" : "=r"(r0), "=r"(r1) : "r"(addr));
}
SK_DEV void nl_mma(float (&d)[4], uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3, uint32_t b0, uint32_t b1) {
    asm volatile(
        "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0, %1, %2, %3}, {%4, %5, %6, %7}, {%8, %9}, "
        "{%0, %1, %2, %3};"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
        : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}
SK_DEV float nl_lif(float U, float I, float o, float lam, float th) {  // Eq.1, no FMA (oracle order)
    return __fsub_rn(__fadd_rn(__fmul_rn(lam, U), I), o != 0.f ? th : 0.f);  // theta * o, o in {0, 1}: exact select
}
}  // namespace

template <int CIN, int N, int S>
__global__ void __launch_bounds__(NL_THREADS, N == 16 ? 3 : 2) narrow_lif_kernel(const NarrowConvArgs a, int TH) {
    pdl_enter();
    extern __shared__ __align__(16) uint8_t smem[];
    const int Hin = a.Hin, Win = a.Win;
    const int RX = S * (TH - 1) + 3;                       // staged input rows per band
    const int XBUF = RX * Win * CIN;                       // bf16 elements of one staging buffer
    // resident weights [9][N][WP]: row pitch WP = CIN + 8 (48 bytes for CIN = 16), so the 8 output-channel
    // rows an ldmatrix reads land in 8 distinct 16-byte bank groups (the [N][9][CIN] layout was 2-way)
    constexpr int WP = CIN + 8;
    uint16_t *sW = reinterpret_cast<uint16_t *>(smem);
    uint16_t *sX = sW + 9 * N * WP;                        // 2 x [RX][Win][CIN] (stride 1: chunk-swizzled)
    uint16_t *sZ = sX + 2 * (size_t)XBUF;                  // zero row [CIN]
    float *sI = reinterpret_cast<float *>(sZ + CIN);      // [NL_P][N + 1] currents of the row
    constexpr int IP = N + 1;                              // padded pitch (conflict-free column writes)
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    for (int i = threadIdx.x; i < N * 9 * CIN / 8; i += NL_THREADS) {  // Wk [N][9][CIN] -> [9][N][WP]
        const int co = i / (9 * CIN / 8), rem = i - co * (9 * CIN / 8), tap = rem / (CIN / 8), cc = rem % (CIN / 8);
        *reinterpret_cast<uint4 *>(sW + (tap * N + co) * WP + cc * 8) = __ldg(reinterpret_cast<const uint4 *>(a.Wk) + i);
    }
    if (threadIdx.x < CIN / 8) reinterpret_cast<uint4 *>(sZ)[threadIdx.x] = make_uint4(0u, 0u, 0u, 0u);

    const long long HW = (long long)a.H * a.W;
    const long long M = (long long)a.nb * HW;               // output pixels per row
    const int tiles = (int)(M / NL_P);
    const int R = a.R;
    const int r_mma0 = a.restore ? 1 : 0;
    const long long in_row = (long long)a.nb * Hin * Win * CIN;
    const uint32_t sW_a = smem_u32(sW), sX_a = smem_u32(sX), sZ_a = smem_u32(sZ);
    // CIN = 16: a staged pixel is two 16-byte chunks; chunk k of pixel q sits at chunk slot
    // 2q + (k ^ ((q >> 2) & 1)), so ANY 8 consecutive pixels' chunk k (the rows of one ldmatrix 8x8 matrix,
    // whatever the tap shift) fall in 8 distinct bank groups - unswizzled the 32-byte pixel pitch made them
    // 2-way conflicting (ncu: 48 % of the shared-load wavefronts excessive)
    // (stride 2 reads every other pixel: the swizzle halves that 4-way conflict to 2-way)
    auto xswz = [&](int c) -> int { return c ^ ((c >> 3) & (CIN / 8 - 1)); };   // chunk index c = (CIN/8) q + k
    const int P = TH * a.W;                                  // == NL_P

    for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
        const long long m0 = (long long)tile * NL_P;
        const long long n = m0 / HW;
        const int y0 = (int)((m0 - n * HW) / a.W);
        auto stage = [&](int r, int b) {  // input rows of timestep row r for this band into buffer b
            const uint32_t dst = sX_a + (uint32_t)(b * XBUF) * 2u;
            const int rowv = Win * CIN / 8;
            const uint16_t *Xr = a.X + (long long)r * in_row;
            for (int i = threadIdx.x; i < RX * rowv; i += NL_THREADS) {
                const int rr = i / rowv, e = i - rr * rowv;
                const int yi = S * y0 - 1 + rr;
                const bool in = yi >= 0 && yi < Hin;
                const uint4 *src = reinterpret_cast<const uint4 *>(Xr + ((n * Hin + (in ? yi : 0)) * (long long)Win) * CIN) + e;
                cp_async16_cg(dst + 16u * (uint32_t)xswz(i), src, in ? 16u : 0u);
            }
            cp_async_commit();
        };
        // ---- epilogue state (threads 0..127 own one pixel each)
        const bool epi = threadIdx.x < NL_P;
        const long long m = m0 + (epi ? threadIdx.x : 0);
        const long long nidx = m * N;
        constexpr int NW = (N + 31) / 32;
        float U[N];
        uint32_t ob[NW];
#pragma unroll
        for (int j = 0; j < NW; ++j) ob[j] = 0u;
        if (epi) {
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
        long long roff = -1, rrs = 0;
        if (a.res && epi) {
            const int y = (int)((m / a.W) % a.H), x = (int)(m % a.W);
            rrs = (long long)a.nb * a.res_H * a.res_W * a.res_C;
            roff = ((n * a.res_H + (long long)y * a.res_stride) * a.res_W + (long long)x * a.res_stride) * a.res_C;
        }
        const long long rs = M * N;
        auto bitf = [&](int c) { return (float)((ob[c >> 5] >> (c & 31)) & 1u); };
        auto store_state = [&](float *Ud, uint8_t *od) {
#pragma unroll
            for (int c = 0; c < N; c += 4) {
                *reinterpret_cast<float4 *>(Ud + c) = make_float4(U[c], U[c + 1], U[c + 2], U[c + 3]);
                const uint32_t w = ob[c >> 5] >> (c & 31);
                *reinterpret_cast<uchar4 *>(od + c) = make_uchar4(w & 1u, (w >> 1) & 1u, (w >> 2) & 1u, (w >> 3) & 1u);
            }
        };
        auto emit = [&](int r, bool counted) {  // warps 0..3 only (all lanes)
            const long long t = a.row_t ? (long long)a.row_t[r] : (long long)a.t0 + r;
            unsigned cnt = 0;
            double q2 = 0.0;
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
            if (a.cnt) {
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
            if (counted && a.s_part) {
                const unsigned v = __reduce_add_sync(0xffffffffu, cnt);
                if (lane == 0 && v) atomicAdd(a.s_part + t * 32 + (blockIdx.x & 31), v);
            }
            if (counted && a.u2_part) u2_warp_add(a.u2_part, t, q2);
        };
        if (a.restore && epi) emit(0, false);

        // this lane's A-row byte offset in a staging buffer for each tap (or ~0u: the zero padding row) - the
        // same for every row of the tile, so the bounds checks and address math leave the row loop
        uint32_t aoff[9][CIN / 16];
        {
            const int pa = warp * 16 + (lane & 7) + ((lane >> 3) & 1) * 8;
            const int ya = pa / a.W, xa = pa - ya * a.W;
            const int kh = (lane >> 4) * 8;
#pragma unroll
            for (int tap = 0; tap < 9; ++tap) {
                const int dy = tap / 3, dx = tap % 3;
                const int xs = S * xa + dx - 1, ys = S * ya + dy;
                const int yi = S * y0 - 1 + ys;
                const bool ok = xs >= 0 && xs < Win && yi >= 0 && yi < Hin;
#pragma unroll
                for (int ks = 0; ks < CIN / 16; ++ks)  // K step ks = channels 16 ks .. 16 ks + 15 (chunks 2 ks, 2 ks + 1)
                    aoff[tap][ks] = ok ? 16u * (uint32_t)xswz((ys * Win + xs) * (CIN / 8) + 2 * ks + kh / 8) : ~0u;
            }
        }
        if (r_mma0 < R) stage(r_mma0, 0);
        int b = 0;
        for (int r = r_mma0; r < R; ++r, b ^= 1) {
            if (r + 1 < R) {
                stage(r + 1, b ^ 1);
                cp_async_wait<1>();
            } else {
                cp_async_wait<0>();
            }
            __syncthreads();  // row r staged; the previous row's currents consumed
            // ---- currents: warp w -> pixels 16w .. 16w+15 of the band, all N channels
            if (warp * 16 < P) {
                float acc[N / 8][4];
#pragma unroll
                for (int j = 0; j < N / 8; ++j) acc[j][0] = acc[j][1] = acc[j][2] = acc[j][3] = 0.f;
                const uint32_t xb = sX_a + (uint32_t)(b * XBUF) * 2u;
                const uint32_t zrow = sZ_a + (uint32_t)((lane >> 4) * 8) * 2u;
                static_assert(CIN == 16 || CIN == 32, "16-channel K steps per tap");
#pragma unroll
                for (int tap = 0; tap < 9; ++tap) {
#pragma unroll
                    for (int ks = 0; ks < CIN / 16; ++ks) {
                        uint32_t a0, a1, a2, a3;
                        nl_ldsm_x4(aoff[tap][ks] != ~0u ? xb + aoff[tap][ks] : zrow, a0, a1, a2, a3);
#pragma unroll
                        for (int nt = 0; nt < N / 8; ++nt) {
                            uint32_t b0, b1;
                            const int co = nt * 8 + (lane & 7), ci = ks * 16 + ((lane >> 3) & 1) * 8;
                            nl_ldsm_x2(sW_a + (uint32_t)((tap * N + co) * WP + ci) * 2u, b0, b1);
                            nl_mma(acc[nt], a0, a1, a2, a3, b0, b1);
                        }
                    }
                }
                const int p0 = warp * 16 + (lane >> 2), c0 = 2 * (lane & 3);
#pragma unroll
                for (int nt = 0; nt < N / 8; ++nt) {
                    sI[p0 * IP + nt * 8 + c0] = acc[nt][0];
                    sI[p0 * IP + nt * 8 + c0 + 1] = acc[nt][1];
                    sI[(p0 + 8) * IP + nt * 8 + c0] = acc[nt][2];
                    sI[(p0 + 8) * IP + nt * 8 + c0 + 1] = acc[nt][3];
                }
            }
            __syncthreads();  // currents of row r in sI; buffer b free for row r + 2
            if (epi) {
                float I[N];
#pragma unroll
                for (int c = 0; c < N; ++c) I[c] = sI[threadIdx.x * IP + c];
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
                    U[c] = nl_lif(U[c], I[c], bitf(c), a.lam, a.theta);
                    nb[c >> 5] |= (U[c] > a.theta ? 1u : 0u) << (c & 31);
                }
#pragma unroll
                for (int j = 0; j < NW; ++j) ob[j] = nb[j];
                emit(r, true);
                if (a.ckU && (a.ck_every ? r % a.ck_every == 0 : r == 0)) {
                    const long long slot = a.ck_every ? (long long)(r / a.ck_every) * a.ck_stride : 0;
                    store_state(a.ckU + slot + nidx, a.cko + slot + nidx);
                }
            }
        }
        if (epi && !a.restore) store_state(a.U_state + nidx, a.o_state + nidx);
        __syncthreads();  // sI / staging buffers reused by the next tile
    }
}

bool narrow_lif_mma_supported(int cin, int cout, int stride, int H, int W) {
    // 32 -> 32 (stride 1): two 16-channel K steps per tap; with the conflict-free staging it beats
    // conv_narrow.cu's tcgen05 gather kernel (cfg 4 SKIP 428.7 -> 444.7 samples/s; round 1, before the
    // swizzled staging, it measured slower).  SKIPPER_NO_NL32=1 restores the gather kernel.
    const char *e = getenv("SKIPPER_NO_NL32");  // read per call so tests can cover both paths in one process
    const bool nl32 = !(e && atoi(e));
    const bool c32 = nl32 && cin == 32 && cout == 32 && stride == 1;
    if (!(c32 || (cin == 16 && (cout == 16 || cout == 32) && (stride == 1 || stride == 2)))) return false;
    if (W > NL_P || NL_P % W || W % 16) return false;
    const int TH = NL_P / W;
    return H % TH == 0 && TH <= H;
}

template <int CIN, int N, int S>
static cudaError_t launch_nl(const NarrowConvArgs &a, cudaStream_t s, int num_sms) {
    const int TH = NL_P / a.W;
    const int RX = S * (TH - 1) + 3;
    const size_t smem = (size_t)9 * N * (CIN + 8) * 2 + 2 * (size_t)RX * a.Win * CIN * 2 + CIN * 2 + (size_t)NL_P * (N + 1) * 4;
    auto kern = narrow_lif_kernel<CIN, N, S>;
    static bool attr = false;
    if (!attr) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
        if (e != cudaSuccess) return e;
        attr = true;
    }
    int per_sm = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, NL_THREADS, smem) != cudaSuccess || per_sm < 1)
        per_sm = 1;
    const long long tiles = (long long)a.nb * a.H * a.W / NL_P;
    if (tiles == 0) return cudaSuccess;
    const int grid = (int)std::min<long long>(tiles, (long long)num_sms * per_sm);
    if (getenv("SKIPPER_NARROW_DEBUG"))
        fprintf(stderr, "[narrow_lif_mma] cin=%d N=%d s=%d smem=%zu per_sm=%d grid=%d tiles=%lld\n", CIN, N, S, smem, per_sm,
                grid, tiles);
    sk_launch(kern, grid, NL_THREADS, smem, s, a, TH);
    return cudaGetLastError();
}

cudaError_t launch_narrow_lif_mma(const NarrowConvArgs &a, cudaStream_t s, int num_sms) {
    if (!narrow_lif_mma_supported(a.Cin, a.Cout, a.stride, a.H, a.W) || a.R <= 0) return cudaErrorInvalidValue;
    if (a.res && (a.res_C % 8 || a.res_lo % 8 || a.res_lo < 0 || a.res_lo + a.res_C > a.Cout)) return cudaErrorInvalidValue;
    if (a.Cin == 32) return launch_nl<32, 32, 1>(a, s, num_sms);
    if (a.Cout == 16 && a.stride == 1) return launch_nl<16, 16, 1>(a, s, num_sms);
    if (a.Cout == 32 && a.stride == 1) return launch_nl<16, 32, 1>(a, s, num_sms);
    if (a.Cout == 16 && a.stride == 2) return launch_nl<16, 16, 2>(a, s, num_sms);
    if (a.Cout == 32 && a.stride == 2) return launch_nl<16, 32, 2>(a, s, num_sms);
    return cudaErrorInvalidValue;
}

}  // namespace sk
