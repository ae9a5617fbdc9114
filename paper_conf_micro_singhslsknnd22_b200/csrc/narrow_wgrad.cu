// narrow_wgrad.cu - weight gradient of the narrow-channel (16 / 32 input channels) 3x3 convolutions of
// the ResNet-DVS SNN (cfg 4), stride 1 or 2, without a column buffer:
//     dW[co][tap][ci] += sum_p delta[p][co] * X[src(p, tap)][ci]          (Eq.2 weight term)
// over every output pixel p of the segment's kept rows.  The explicit path (im2col of 18-36 B per
// input pixel per tap into HBM, then a GEMM over the columns) moved ~9x the layer input through HBM;
// here each CTA stages one (image, band of output rows) unit in shared memory - the delta tile and
// the input rows it reads, zero rows for the padding; cp.async, double-buffered so the next unit
// streams in while this one computes - and its warps run bf16 m16n8k16 tensor-core
// MMAs whose B operand rows are gathered by ldmatrix straight from the staged input (one row address
// per output pixel and tap, so the shift / stride / zero padding costs nothing).  The work is
// bandwidth-sized (K = pixels, M = cout, N = 9 cin), so the warp-level MMA is not the bound; the
// accumulators stay in registers across all units of a persistent CTA and are reduced once at the end,
// in a fixed order (warps in turn into shared memory, then the CTA's own dW slice; the slices are summed in
// slice order by launch_reduce_slices), so the weight gradient is deterministic.
#include "common.cuh"
#include "kernels.h"

#include <algorithm>

namespace sk {

namespace {

constexpr int NW_THREADS = 256;
constexpr int NW_P = 128;  // output pixels per unit

template <int CIN, int COUT>
struct NwCfg {
    static constexpr int MT = COUT / 16;                   // M tiles of 16 output channels
    static constexpr int NTT = CIN / 8;                    // n tiles of 8 input channels per tap
    static constexpr int NTG = CIN == 16 ? (MT == 4 ? 2 : 1) : 8 / MT;  // tap groups
    static constexpr int COMBOS = MT * NTG;                // (M tile, tap group) work items
    static constexpr int WPC = 8 / COMBOS;                 // warps per work item (split over k chunks)
    static constexpr int MAXT = (9 + NTG - 1) / NTG;       // taps per group (max)
    static_assert(8 % COMBOS == 0, "work items must divide the 8 warps");
};

// Staged [pixel][C] bf16 rows are ldmatrix'ed as 8 consecutive pixels' 16-byte chunk k.  With CP = C / 8
// chunks per pixel that is 8 rows at a CP x 16-byte pitch: 2- (C = 16), 4- (32) or 8-way (64) bank conflicts.
// Chunk c (= CP * pixel + k) is stored at slot c ^ ((c >> 3) & (CP - 1)): the 8 rows of any 8 consecutive
// pixels land in 8 distinct 16-byte bank groups.
template <int C>
SK_DEV uint32_t xswz(uint32_t c) {
    return c ^ ((c >> 3) & (uint32_t)(C / 8 - 1));
}

SK_DEV void ldsm_x4_t(uint32_t addr, uint32_t &r0, uint32_t &r1, uint32_t &r2, uint32_t &r3) {
    asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0, %1, %2, %3}, [%4];"
                 : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3)
                 : "r"(addr));
}
SK_DEV void ldsm_x2_t(uint32_t addr, uint32_t &r0, uint32_t &r1) {
    asm volatile("ldmatrix.sync.aligned.m8n8.x2.trans.shared.b16 {%0, %1}, [%2];" : "=r"(r0), "=r"(r1) : "r"(addr));
}
SK_DEV void mma_bf16(float (&d)[4], uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3, uint32_t b0, uint32_t b1) {
    asm volatile(
        "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0, %1, %2, %3}, {%4, %5, %6, %7}, {%8, %9}, "
        "{%0, %1, %2, %3};"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
        : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}

}  // namespace

// X [nb][Hin][Win][CIN] bf16, D [nb][H][W][COUT] bf16 (H = Hin / S), dW [COUT][9][CIN] fp32 (+=)
template <int CIN, int COUT, int S>
__global__ void __launch_bounds__(NW_THREADS) narrow_wgrad_kernel(const uint16_t *__restrict__ X,
                                                                   const uint16_t *__restrict__ D, float *dW, int nb,
                                                                   int H, int W, int TH) {
    pdl_enter();
    using Cfg = NwCfg<CIN, COUT>;
    extern __shared__ __align__(16) uint8_t smem[];
    const int Hin = H * S, Win = W * S;
    const int RX = S * (TH - 1) + 3;                      // staged input rows per unit
    const int BUF = NW_P * COUT + RX * Win * CIN;         // bf16 elements of one staging buffer
    uint16_t *sB = reinterpret_cast<uint16_t *>(smem);    // 2 x { delta [NW_P][COUT], input [RX][Win][CIN] }
    uint16_t *sZ = sB + 2 * (size_t)BUF;                  // one zero row [CIN]
    float *sR = reinterpret_cast<float *>(sZ + CIN);      // [COUT * 9 * CIN] cross-warp reduction (WPC > 1)
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int combo = warp / Cfg::WPC, wk = warp % Cfg::WPC;
    const int mt = combo / Cfg::NTG, tg = combo % Cfg::NTG;
    const int tap0 = tg * 9 / Cfg::NTG, tap1 = (tg + 1) * 9 / Cfg::NTG;
    if (threadIdx.x < CIN / 8) reinterpret_cast<uint4 *>(sZ)[threadIdx.x] = make_uint4(0u, 0u, 0u, 0u);
    if (Cfg::WPC > 1)
        for (int i = threadIdx.x; i < COUT * 9 * CIN; i += NW_THREADS) sR[i] = 0.f;

    float acc[Cfg::MAXT][Cfg::NTT][4];
#pragma unroll
    for (int t = 0; t < Cfg::MAXT; ++t)
#pragma unroll
        for (int j = 0; j < Cfg::NTT; ++j) acc[t][j][0] = acc[t][j][1] = acc[t][j][2] = acc[t][j][3] = 0.f;

    const int bands = H / TH;
    const long long units = (long long)nb * bands;
    const uint32_t sB_a = smem_u32(sB), sZ_a = smem_u32(sZ);
    // stage unit u into buffer b with cp.async (16-byte pieces; rows outside the image are zero-filled)
    auto stage = [&](long long u, int b) {
        const long long n = u / bands;
        const int y0 = (int)(u - n * bands) * TH;
        const uint32_t dD = sB_a + (uint32_t)(b * BUF) * 2u, dX = dD + (uint32_t)(NW_P * COUT) * 2u;
        const uint4 *src = reinterpret_cast<const uint4 *>(D + ((n * H + y0) * (long long)W) * COUT);
        const int nD = TH * W * COUT / 8;
        for (int i = threadIdx.x; i < nD; i += NW_THREADS) cp_async16_cg(dD + 16u * xswz<COUT>(i), src + i, 16u);
        const int rowv = Win * CIN / 8;
        const int nX = RX * rowv;
        for (int i = threadIdx.x; i < nX; i += NW_THREADS) {
            const int r = i / rowv, e = i - r * rowv;
            const int yi = S * y0 - 1 + r;
            const bool in = yi >= 0 && yi < Hin;
            const uint4 *xs = reinterpret_cast<const uint4 *>(X + ((n * Hin + (in ? yi : 0)) * (long long)Win) * CIN) + e;
            cp_async16_cg(dX + 16u * xswz<CIN>(i), xs, in ? 16u : 0u);
        }
        cp_async_commit();
    };
    if ((long long)blockIdx.x < units) stage(blockIdx.x, 0);
    int b = 0;
    for (long long u = blockIdx.x; u < units; u += gridDim.x, b ^= 1) {
        const long long n = u / bands;
        const int y0 = (int)(u - n * bands) * TH;
        const long long un = u + gridDim.x;
        if (un < units) {
            stage(un, b ^ 1);   // the buffer the previous unit read (released by the barrier below)
            cp_async_wait<1>(); // this unit's pieces have landed (the next unit's may still be in flight)
        } else {
            cp_async_wait<0>();
        }
        __syncthreads();
        const uint32_t sD_a = sB_a + (uint32_t)(b * BUF) * 2u, sX_a = sD_a + (uint32_t)(NW_P * COUT) * 2u;
        const int P = TH * W;
        for (int kc = wk; kc < P / 16; kc += Cfg::WPC) {
            // A = delta^T (m = output channel, k = pixel): 4 transposed 8x8 blocks of the delta tile
            uint32_t a0, a1, a2, a3;
            {
                const int j = lane >> 3, r = lane & 7;
                const int k = kc * 16 + ((j & 2) ? 8 : 0) + r;
                const int m = mt * 16 + ((j & 1) ? 8 : 0);
                ldsm_x4_t(sD_a + 16u * xswz<COUT>((uint32_t)(k * (COUT / 8) + m / 8)), a0, a1, a2, a3);
            }
            // this lane's B row: output pixel kc*16 + (lane & 15)
            const int p = kc * 16 + (lane & 15);
            const int yl = p / W, x = p - yl * W;
#pragma unroll
            for (int t = 0; t < Cfg::MAXT; ++t) {
                const int tap = tap0 + t;
                if (tap >= tap1) break;
                const int dy = tap / 3, dx = tap % 3;
                const int xs = S * x + dx - 1;
                const int ys = S * yl + dy;                       // staged row
                const int yi = S * y0 - 1 + ys;                   // image row
                const bool ok = xs >= 0 && xs < Win && yi >= 0 && yi < Hin;
                const uint32_t c0 = (uint32_t)((ys * Win + xs) * (CIN / 8));
#pragma unroll
                for (int j = 0; j < Cfg::NTT; ++j) {
                    uint32_t b0, b1;
                    ldsm_x2_t(ok ? sX_a + 16u * xswz<CIN>(c0 + j) : sZ_a + (uint32_t)j * 16u, b0, b1);
                    mma_bf16(acc[t][j], a0, a1, a2, a3, b0, b1);
                }
            }
        }
        __syncthreads();  // buffer b is free for the unit after next
    }
    // D fragment: rows (co) mt*16 + lane/4 (+8), cols (ci within n tile) 2*(lane%4) (+1)
    // Deterministic reduction: the WPC warps of a work item add their partials into sR in turn (wk order),
    // then the CTA adds its sum into its own slice dW + blockIdx.x * |dW| - one writer per slice per launch,
    // launches in stream order - and launch_reduce_slices sums the slices in slice order.
    const int co = mt * 16 + (lane >> 2), ci0 = 2 * (lane & 3);
    float *dst = dW + (size_t)blockIdx.x * (COUT * 9 * CIN);
    if (Cfg::WPC > 1) {
        __syncthreads();
        for (int turn = 0; turn < Cfg::WPC; ++turn) {
            if (wk == turn) {
#pragma unroll
                for (int t = 0; t < Cfg::MAXT; ++t) {
                    const int tap = tap0 + t;
                    if (tap >= tap1) break;
#pragma unroll
                    for (int j = 0; j < Cfg::NTT; ++j) {
                        const int ci = j * 8 + ci0;
                        sR[(co * 9 + tap) * CIN + ci] += acc[t][j][0];
                        sR[(co * 9 + tap) * CIN + ci + 1] += acc[t][j][1];
                        sR[((co + 8) * 9 + tap) * CIN + ci] += acc[t][j][2];
                        sR[((co + 8) * 9 + tap) * CIN + ci + 1] += acc[t][j][3];
                    }
                }
            }
            __syncthreads();
        }
        for (int i = threadIdx.x; i < COUT * 9 * CIN; i += NW_THREADS)
            if (sR[i] != 0.f) dst[i] += sR[i];
    } else {  // every element has one owner (warp, lane) in the CTA
#pragma unroll
        for (int t = 0; t < Cfg::MAXT; ++t) {
            const int tap = tap0 + t;
            if (tap >= tap1) break;
#pragma unroll
            for (int j = 0; j < Cfg::NTT; ++j) {
                const int ci = j * 8 + ci0;
                dst[(co * 9 + tap) * CIN + ci] += acc[t][j][0];
                dst[(co * 9 + tap) * CIN + ci + 1] += acc[t][j][1];
                dst[((co + 8) * 9 + tap) * CIN + ci] += acc[t][j][2];
                dst[((co + 8) * 9 + tap) * CIN + ci + 1] += acc[t][j][3];
            }
        }
    }
}

namespace {
SK_DEV void ldsm_x4(uint32_t addr, uint32_t &r0, uint32_t &r1, uint32_t &r2, uint32_t &r3) {
    asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0, %1, %2, %3}, [%4];"
                 : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3)
                 : "r"(addr));
}
SK_DEV void ldsm_x2(uint32_t addr, uint32_t &r0, uint32_t &r1) {
    asm volatile("ldmatrix.sync.aligned.m8n8.x2.shared.b16 {%0, %1}, [%2];" : "=r"(r0), "=r"(r1) : "r"(addr));
}
}  // namespace

// dgrad of a narrow 3x3 conv, stride S in {1, 2} (Eq.2's g = W^T delta):
//     G[n, yi, xi, ci] = sum_{dy, dx, co} W[co][dy*3+dx][ci] D[n, (yi+1-dy)/S, (xi+1-dx)/S, co]
// (terms whose (yi+1-dy, xi+1-dx) is not a multiple of S or leaves the image vanish).  M = pixels of a
// band of G (8 warps x 16), N = ci, K = (tap, co).  The delta rows the band reads are staged by cp.async
// (double-buffered), the transposed weights Wt [ci][9][co] stay resident, and the A rows (one per pixel
// and tap, or a zero row) are gathered by ldmatrix.  Replaces conv_narrow's dgrad (S = 1) and the
// GEMM-into-columns + col2im of the stride-2 layers.
template <int CI, int CO, int S>
__global__ void __launch_bounds__(NW_THREADS) narrow_dgrad_kernel(const uint16_t *__restrict__ D,
                                                                   const uint16_t *__restrict__ Wt, float *G, int nb,
                                                                   int H, int W, int TH) {
    pdl_enter();
    extern __shared__ __align__(16) uint8_t smem[];
    const int Hg = S * H, Wg = S * W;                     // G (layer input) size
    const int RD = TH / S + 2;                            // staged delta rows per band (max)
    const int BUF = RD * W * CO;                          // bf16 elements of one staging buffer
    constexpr int WP = CO + 8;                            // weight row pitch: conflict-free ldmatrix rows
    uint16_t *sW = reinterpret_cast<uint16_t *>(smem);   // [9][CI][WP]
    uint16_t *sB = sW + 9 * CI * WP;                      // 2 x [RD][W][CO] (chunk-swizzled)
    uint16_t *sZ = sB + 2 * (size_t)BUF;                  // zero row [CO]
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    for (int i = threadIdx.x; i < 9 * CI * CO / 8; i += NW_THREADS) {  // Wt [CI][9][CO] -> [9][CI][WP]
        const int ci = i / (9 * CO / 8), rem = i - ci * (9 * CO / 8), tap = rem / (CO / 8), cc = rem % (CO / 8);
        *reinterpret_cast<uint4 *>(sW + (tap * CI + ci) * WP + cc * 8) = __ldg(reinterpret_cast<const uint4 *>(Wt) + i);
    }
    if (threadIdx.x < CO / 8) reinterpret_cast<uint4 *>(sZ)[threadIdx.x] = make_uint4(0u, 0u, 0u, 0u);
    const int bands = Hg / TH;
    const long long units = (long long)nb * bands;
    const uint32_t sW_a = smem_u32(sW), sB_a = smem_u32(sB), sZ_a = smem_u32(sZ);
    auto fdiv = [](int a) { return a >= 0 ? a / S : -((-a + S - 1) / S); };  // floor(a / S)
    auto stage = [&](long long u, int b) {
        const long long n = u / bands;
        const int y0 = (int)(u - n * bands) * TH;
        const int ylo = fdiv(y0 - 1);
        const uint32_t dst = sB_a + (uint32_t)(b * BUF) * 2u;
        const int rowv = W * CO / 8;
        for (int i = threadIdx.x; i < RD * rowv; i += NW_THREADS) {
            const int r = i / rowv, e = i - r * rowv;
            const int y = ylo + r;
            const bool in = y >= 0 && y < H;
            const uint4 *src = reinterpret_cast<const uint4 *>(D + ((n * H + (in ? y : 0)) * (long long)W) * CO) + e;
            cp_async16_cg(dst + 16u * xswz<CO>(i), src, in ? 16u : 0u);
        }
        cp_async_commit();
    };
    if ((long long)blockIdx.x < units) stage(blockIdx.x, 0);
    int b = 0;
    for (long long u = blockIdx.x; u < units; u += gridDim.x, b ^= 1) {
        const long long n = u / bands;
        const int y0 = (int)(u - n * bands) * TH;
        const int ylo = fdiv(y0 - 1);
        const long long un = u + gridDim.x;
        if (un < units) {
            stage(un, b ^ 1);
            cp_async_wait<1>();
        } else {
            cp_async_wait<0>();
        }
        __syncthreads();
        const uint32_t sD_a = sB_a + (uint32_t)(b * BUF) * 2u;
        if (warp * 16 < TH * Wg) {
            float acc[CI / 8][4];
#pragma unroll
            for (int j = 0; j < CI / 8; ++j) acc[j][0] = acc[j][1] = acc[j][2] = acc[j][3] = 0.f;
            // this lane's A row: G pixel warp*16 + (lane&7) + ((lane>>3)&1)*8, k half (lane>>4)*8
            const int pa = warp * 16 + (lane & 7) + ((lane >> 3) & 1) * 8;
            const int ya = pa / Wg, xa = pa - ya * Wg;
            const int kh = (lane >> 4) * 8;
#pragma unroll
            for (int tap = 0; tap < 9; ++tap) {
                const int dy = tap / 3, dx = tap % 3;
                const int ty = y0 + ya + 1 - dy, tx = xa + 1 - dx;  // S * (delta pixel) when it exists
                const int ys = fdiv(ty), xs = fdiv(tx);
                const bool ok = ys * S == ty && xs * S == tx && ys >= 0 && ys < H && xs >= 0 && xs < W;
                const uint32_t c0 = (uint32_t)(((ys - ylo) * W + xs) * (CO / 8));
#pragma unroll
                for (int ks = 0; ks < CO / 16; ++ks) {
                    uint32_t a0, a1, a2, a3;
                    ldsm_x4(ok ? sD_a + 16u * xswz<CO>(c0 + (ks * 16 + kh) / 8) : sZ_a + (uint32_t)(ks * 16 + kh) * 2u, a0,
                            a1, a2, a3);
#pragma unroll
                    for (int nt = 0; nt < CI / 8; ++nt) {
                        uint32_t b0, b1;
                        const int ci = nt * 8 + (lane & 7), co = ks * 16 + ((lane >> 3) & 1) * 8;
                        ldsm_x2(sW_a + (uint32_t)((tap * CI + ci) * WP + co) * 2u, b0, b1);
                        mma_bf16(acc[nt], a0, a1, a2, a3, b0, b1);
                    }
                }
            }
            // D fragment: pixel warp*16 + lane/4 (+8), ci nt*8 + 2*(lane%4) (+1)
            const int p0 = warp * 16 + (lane >> 2);
#pragma unroll
            for (int h2 = 0; h2 < 2; ++h2) {
                const int p = p0 + 8 * h2;
                const int yy = y0 + p / Wg, xx = p % Wg;
                float *dst = G + (((n * Hg + yy) * (long long)Wg + xx) * CI) + 2 * (lane & 3);
#pragma unroll
                for (int nt = 0; nt < CI / 8; ++nt)
                    *reinterpret_cast<float2 *>(dst + nt * 8) = make_float2(acc[nt][2 * h2], acc[nt][2 * h2 + 1]);
            }
        }
        __syncthreads();
    }
}

// H x W is the delta (output) size; G is (S*H) x (S*W)
// exactly the (cin, cout, stride) instantiations of launch_narrow_dgrad below: a layer this predicate
// rejects takes the GEMM + col2im branch of the engine instead of failing the step
static bool nd_instantiated(int cin, int cout, int stride) {
    if (stride == 1) return (cin == 16 && (cout == 16 || cout == 32)) || (cin == 32 && (cout == 16 || cout == 32));
    if (stride == 2) return (cin == 16 && (cout == 16 || cout == 32)) || (cin == 32 && (cout == 32 || cout == 64));
    return false;
}

bool narrow_dgrad_supported(int cin, int cout, int H, int W, int stride) {
    if (!nd_instantiated(cin, cout, stride)) return false;
    const int Wg = stride * W, Hg = stride * H;
    if (Wg > NW_P || NW_P % Wg || Wg % 16) return false;
    const int TH = std::min(Hg, NW_P / Wg);
    return Hg % TH == 0 && TH % stride == 0;
}

template <int CI, int CO, int S>
static cudaError_t launch_nd(const uint16_t *D, const uint16_t *Wt, float *G, int nb, int H, int W, cudaStream_t s,
                             int num_sms) {
    const int Hg = S * H, Wg = S * W;
    const int TH = std::min(Hg, NW_P / Wg);
    const size_t smem = (size_t)9 * CI * (CO + 8) * 2 + 2 * (size_t)(TH / S + 2) * W * CO * 2 + CO * 2;
    auto kern = narrow_dgrad_kernel<CI, CO, S>;
    static bool attr = false;
    if (!attr) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
        if (e != cudaSuccess) return e;
        attr = true;
    }
    int per_sm = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, NW_THREADS, smem) != cudaSuccess || per_sm < 1)
        per_sm = 1;
    const long long units = (long long)nb * (Hg / TH);
    if (units == 0) return cudaSuccess;
    const int grid = (int)std::min<long long>(units, (long long)num_sms * per_sm);
    sk_launch(kern, grid, NW_THREADS, smem, s, D, Wt, G, nb, H, W, TH);
    return cudaGetLastError();
}

// G [nb][S*H][S*W][cin] fp32 = dgrad of D [nb][H][W][cout] through Wt [cin][9][cout] (bf16)
cudaError_t launch_narrow_dgrad(const uint16_t *D, const uint16_t *Wt, float *G, int nb, int H, int W, int cin, int cout,
                                int stride, cudaStream_t s, int num_sms) {
    if (!narrow_dgrad_supported(cin, cout, H, W, stride)) return cudaErrorInvalidValue;
#define ND_CASE(CI_, CO_, S_) \
    if (cin == CI_ && cout == CO_ && stride == S_) return launch_nd<CI_, CO_, S_>(D, Wt, G, nb, H, W, s, num_sms)
    ND_CASE(16, 16, 1);
    ND_CASE(16, 32, 1);
    ND_CASE(32, 16, 1);
    ND_CASE(32, 32, 1);
    ND_CASE(16, 16, 2);
    ND_CASE(16, 32, 2);
    ND_CASE(32, 32, 2);
    ND_CASE(32, 64, 2);
#undef ND_CASE
    return cudaErrorInvalidValue;
}

bool narrow_wgrad_supported(int cin, int cout, int stride, int H, int W) {
    if (!((cin == 16 || cin == 32) && (cout == 16 || cout == 32 || cout == 64) && (stride == 1 || stride == 2)))
        return false;
    if (W > NW_P || NW_P % W || W % 16) return false;  // 16-pixel k chunks inside one image row band
    const int TH = std::min(H, NW_P / W);
    return H % TH == 0;
}

template <int CIN, int COUT, int S>
static size_t nw_smem(int H, int W) {
    using Cfg = NwCfg<CIN, COUT>;
    const int TH = std::min(H, NW_P / W);
    const int RX = S * (TH - 1) + 3;
    return 2 * ((size_t)NW_P * COUT * 2 + (size_t)RX * W * S * CIN * 2) + CIN * 2 +
           (Cfg::WPC > 1 ? (size_t)COUT * 9 * CIN * 4 : 0);
}

// the persistent grid's size = the number of dW slices (fixed per layer shape, independent of nb)
template <int CIN, int COUT, int S>
static int nw_grid_max(int H, int W, int num_sms) {
    auto kern = narrow_wgrad_kernel<CIN, COUT, S>;
    static bool attr = false;
    if (!attr) {
        if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024) != cudaSuccess)
            return 0;
        attr = true;
    }
    int per_sm = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, NW_THREADS, nw_smem<CIN, COUT, S>(H, W)) !=
            cudaSuccess || per_sm < 1)
        per_sm = 1;
    return num_sms * per_sm;
}

template <int CIN, int COUT, int S>
static cudaError_t launch_nw(const uint16_t *X, const uint16_t *D, float *dW, int nb, int H, int W, cudaStream_t s,
                             int num_sms) {
    const int TH = std::min(H, NW_P / W);
    const size_t smem = nw_smem<CIN, COUT, S>(H, W);
    if (smem > 200 * 1024) return cudaErrorInvalidValue;
    const int gmax = nw_grid_max<CIN, COUT, S>(H, W, num_sms);
    if (gmax < 1) return cudaErrorInvalidValue;
    const long long units = (long long)nb * (H / TH);
    if (units == 0) return cudaSuccess;
    const int grid = (int)std::min<long long>(units, (long long)gmax);
    sk_launch(narrow_wgrad_kernel<CIN, COUT, S>, grid, NW_THREADS, smem, s, X, D, dW, nb, H, W, TH);
    return cudaGetLastError();
}

#define NW_CASES(X_)  \
    X_(16, 16, 1);    \
    X_(16, 32, 1);    \
    X_(16, 64, 1);    \
    X_(32, 16, 1);    \
    X_(32, 32, 1);    \
    X_(32, 64, 1);    \
    X_(16, 16, 2);    \
    X_(16, 32, 2);    \
    X_(16, 64, 2);    \
    X_(32, 16, 2);    \
    X_(32, 32, 2);    \
    X_(32, 64, 2)

int narrow_wgrad_slices(int cin, int cout, int stride, int H, int W, int num_sms) {
    if (!narrow_wgrad_supported(cin, cout, stride, H, W)) return 0;
#define NWS_CASE(CI, CO, ST) \
    if (cin == CI && cout == CO && stride == ST) return nw_grid_max<CI, CO, ST>(H, W, num_sms)
    NW_CASES(NWS_CASE);
#undef NWS_CASE
    return 0;
}

cudaError_t launch_narrow_wgrad(const uint16_t *X, const uint16_t *D, float *dW, int nb, int H, int W, int cin,
                                int cout, int stride, cudaStream_t s, int num_sms) {
    if (!narrow_wgrad_supported(cin, cout, stride, H, W)) return cudaErrorInvalidValue;
#define NW_CASE(CI, CO, ST) \
    if (cin == CI && cout == CO && stride == ST) return launch_nw<CI, CO, ST>(X, D, dW, nb, H, W, s, num_sms)
    NW_CASES(NW_CASE);
#undef NW_CASE
    return cudaErrorInvalidValue;
}

}  // namespace sk
