// conv_lif.cu - K2+K1 fused for 3x3 convolution layers: synaptic current on the tcgen05 tensor cores
// and the LIF recurrence (Eq.1) in the epilogue, so the fp32 currents never reach HBM.
//
// Work unit = (tile of 128 output pixels of one timestep, tile of BN output channels).  A CTA walks the
// rows (timesteps) of its unit in order: for every row the implicit-GEMM K loop (one 3x3 tap x 64
// input channels per K block, 4D TMA box shifted by the tap, zero padding = TMA out-of-bounds fill)
// accumulates I_t into one of two TMEM accumulators; the epilogue warps hold the membrane potentials
// of the unit in registers across rows (thread = pixel, BN/2 channels), apply
//     U_t = ((lam * U_{t-1}) + I_t) - theta * o_{t-1},   o_t = [U_t > theta]      (no FMA, as the oracle)
// and write the layer output (bf16 spikes, or their 2x2 average through a shared-memory exchange),
// the stored membranes (RECORD / RECOMPUTE), the segment checkpoint, the SAM counts (Eq.4)
// and the debug record.  The MMA of row t+1 overlaps the epilogue of row t.
//
//   warp 0      TMA producer            warp 1      MMA issuer + TMEM owner
//   warps 2-9   epilogue: warp w reads TMEM lane quadrant w % 4 (32 pixels), channel half (w - 2) / 4
#include "common.cuh"
#include "gemm.h"

#include <cstdio>
#include <cstdlib>

#ifdef SK_L0_STATS
// diagnostic build (-DSK_L0_STATS): lane 0 of warps 0, 1, 2 of CTA 0 accumulates cycles per section
#define CL_STAT_DECL                               \
    long long cls_[8] = {0, 0, 0, 0, 0, 0, 0, 0}; \
    long long clt_ = 0;                            \
    const long long clk_ = clock64()
#define CL_T0 clt_ = clock64()
#define CL_T1(i) cls_[i] += clock64() - clt_
#define CL_STAT_DUMP                                                                                             \
    if (blockIdx.x == 0 && lane == 0 && warp <= 2)                                                               \
        printf("clstats warp %d total %lld s1 %lld s2 %lld s3 %lld s4 %lld s5 %lld\n", warp, clock64() - clk_, \
               cls_[1], cls_[2], cls_[3], cls_[4], cls_[5])
#else
#define CL_STAT_DECL
#define CL_T0
#define CL_T1(i)
#define CL_STAT_DUMP
#endif

namespace sk {

static constexpr int CL_BM = 128;
static constexpr int CL_BK = 64;
static constexpr int CL_EPI_WARPS = 8;
static constexpr int CL_THREADS = 32 * (2 + CL_EPI_WARPS);
static constexpr int CL_MAXST = 8;  // max smem ring stages
static constexpr uint32_t CL_AH_MAX = 24576;  // halo activation box: (128 / W + 2) * W * 128 B, W <= 32

template <int BN, int PAIR>
struct ClCfg {
    static constexpr uint32_t A_BYTES = CL_BM * CL_BK * 2;
    static constexpr uint32_t B_BYTES = (PAIR ? BN / 2 : BN) * CL_BK * 2;  // this CTA's slice of the weights
    static constexpr uint32_t STAGE_BYTES = A_BYTES + B_BYTES;
    static constexpr int STAGES = STAGE_BYTES <= 24576 ? 8 : 6;  // streamed-weight ring depth
    static constexpr int NACC = 512 / BN < 4 ? 512 / BN : 4;  // TMEM accumulator ring (rows in flight)
    static constexpr uint32_t TMEM_COLS = NACC * BN <= 128 ? 128 : (NACC * BN <= 256 ? 256 : 512);
    static constexpr int CW = BN / 2;                        // channels per epilogue thread
    static constexpr uint32_t SPK_BYTES = 2u * CL_BM * (BN / 32) * 4u;  // 2 buffers of spike words
    static constexpr uint32_t BAR_BYTES = 8 * (2 * CL_MAXST + 10) + 16;
    static constexpr uint32_t FIXED_BYTES = 1024 + SPK_BYTES + BAR_BYTES;  // + stages (+ resident weights)
};

SK_DEV float cl_lif(float U, float I, float o, float lam, float th) {
    return __fsub_rn(__fadd_rn(__fmul_rn(lam, U), I), o != 0.f ? th : 0.f);  // theta * o, o in {0, 1}: exact select
}

// PAIR = 1: a cluster of two CTAs on the two SMs of a TPC runs M = 256 MMAs (tcgen05 cta_group::2):
// each CTA loads its own 128-pixel A tile and half of the weight tile (BN/2 channels) into its own
// shared memory, the leader's MMA reads both halves and writes each CTA's 128 accumulator rows into
// that CTA's TMEM.  Per SM that halves the weight bytes both read by the MMA and written by TMA —
// the kernel is shared-memory-bandwidth bound.  Every CTA runs the same number of unit
// iterations (phantom units past the end load and multiply but write nothing).
// RESB = 1 (pairs only): each CTA keeps its half of the unit's weights resident in shared memory for
// all rows of the unit (loaded once), so the ring streams only activations: per SM the TMA ingress
// per MMA drops from 24 KB to 16 KB per K block (the kernel is bound by per-SM TMA ingress).
// HALO = 1 (single CTA, tiles of whole image rows, W >= 8): per (row, 64-channel block, dx) ONE
// activation box of bh + 2 image rows (the tile plus its vertical halo, zero-filled out of bounds) is
// loaded together with the weights of the three vertical taps; the three dy taps read the same box at
// descriptor offsets of dy * W rows (multiples of the 1024-byte swizzle atom).  Activation boxes per
// row: 3 * Cin/64 instead of 9 * Cin/64 (the kernel is bound by per-SM TMA box processing).
// BWD = 1 / 2 (NEXT-1 backward half, K2 + K4): the same implicit-GEMM mainloop computes the weight-gradient
// input g^{l-1}_t = conv(delta^l_t, W^l flipped) of a stride-1 3x3 layer (A = delta^l rows, taps shifted as in
// the forward, weights [Cin][9][Cout] read at the flipped tap 8 - tap), walking the rows DOWNWARDS, and the
// epilogue runs the reverse surrogate scan of layer l-1 (Eq.2; triangle (1) / fast-sigmoid (2)
// surrogate) on the accumulator:  delta_t = sigma'(U_t) * g_t + lam * delta_{t+1}  (carry in / out), writing
// the bf16 delta rows - g never reaches HBM.
template <int BN, int POOL, int PAIR, int RESB, int HALO, int BWD = 0>
__global__ void __launch_bounds__(CL_THREADS, 1)
    conv_lif_kernel(const __grid_constant__ CUtensorMap ta, const __grid_constant__ CUtensorMap tb, const ConvLifArgs a) {
    pdl_enter();
    using Cfg = ClCfg<BN, PAIR>;
    constexpr int CW = Cfg::CW;
    constexpr int NW = BN / 32;  // spike words per pixel
    const int STAGES = a.stages;
    constexpr uint32_t A_STAGE = HALO ? CL_AH_MAX : Cfg::A_BYTES;                  // activation part of a stage
    constexpr uint32_t SBYTES = A_STAGE + (RESB ? 0u : (HALO ? 3u : 1u) * Cfg::B_BYTES);  // bytes per ring stage
    const int steps = HALO ? 3 * a.conv_cb : a.num_kb;  // ring stages per row
    extern __shared__ uint8_t smem_raw[];
    const uint32_t raw = smem_u32(smem_raw);
    const uint32_t base = (raw + 1023u) & ~1023u;
    const uint32_t bres = base;  // resident weights [num_kb][BN/2 rows][128 B] (RESB)
    const uint32_t sring = base + (RESB ? (uint32_t)a.num_kb * Cfg::B_BYTES : 0u);
    const uint32_t spk = sring + STAGES * SBYTES;
    const uint32_t bars = spk + Cfg::SPK_BYTES;
    auto full_bar = [&](int s) { return bars + 8u * s; };
    auto empty_bar = [&](int s) { return bars + 8u * (CL_MAXST + s); };
    constexpr int NACC = Cfg::NACC;
    auto tfull_bar = [&](int i) { return bars + 8u * (2 * CL_MAXST + i); };
    auto tempty_bar = [&](int i) { return bars + 8u * (2 * CL_MAXST + 4 + i); };
    const uint32_t bfull_bar = bars + 8u * (2 * CL_MAXST + 8);
    const uint32_t bempty_bar = bars + 8u * (2 * CL_MAXST + 9);
    const uint32_t tmem_slot = bars + 8u * (2 * CL_MAXST + 10);
    unsigned *s_cnt = reinterpret_cast<unsigned *>(smem_raw + (tmem_slot + 16 - raw));
    uint32_t *s_spk = reinterpret_cast<uint32_t *>(smem_raw + (spk - raw));

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int r_mma0 = (!BWD && a.restore) ? 1 : 0;
    const int HW = a.H * a.W;
    const int BHW = a.B * HW;
    auto row_of = [&](int r) -> int { return BWD ? a.R - 1 - r : r; };  // backward: rows downwards
    auto wtap = [&](int tap) -> int { return BWD ? 8 - tap : tap; };    // backward: flipped weight taps
    // work decomposition: PAIR -> pair index / rank; unit = (pixel-tile group, channel tile)
    const int rank = PAIR ? (int)cluster_ctarank() : 0;
    const int grp_tiles = PAIR ? a.m_tiles / 2 : a.m_tiles;  // pixel-tile groups per channel tile
    const int units = grp_tiles * a.n_tiles;
    const int wid = PAIR ? (int)blockIdx.x / 2 : (int)blockIdx.x;
    const int nworkers = PAIR ? (int)gridDim.x / 2 : (int)gridDim.x;
    const int niter = (units + nworkers - 1) / nworkers;  // uniform across the grid
    auto unit_tile = [&](int it, int &mt, int &nt) -> bool {
        const int u = wid + it * nworkers;
        mt = (u % grp_tiles) * (PAIR ? 2 : 1) + rank;
        nt = u / grp_tiles;
        return u < units;
    };

    for (int r = threadIdx.x; r < a.R; r += blockDim.x) s_cnt[r] = 0;
    if (threadIdx.x == 0) {
        tma_prefetch(&ta);
        tma_prefetch(&tb);
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(full_bar(s), 1);
            mbar_init(empty_bar(s), 1);
        }
        for (int i = 0; i < NACC; ++i) {
            mbar_init(tfull_bar(i), 1);
            mbar_init(tempty_bar(i), CL_EPI_WARPS * (PAIR ? 2 : 1));  // epilogue warps of both CTAs
        }
        mbar_init(bfull_bar, 1);
        mbar_init(bempty_bar, 1);
        fence_mbar_init();
    }
    if (warp == 1) {
        if (PAIR)
            tmem_alloc_2sm<Cfg::TMEM_COLS>(tmem_slot);
        else
            tmem_alloc<Cfg::TMEM_COLS>(tmem_slot);
    }
    tc_fence_before();
    if (PAIR)
        cluster_sync_all();
    else
        __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *reinterpret_cast<volatile uint32_t *>(smem_raw + (tmem_slot - raw));
    CL_STAT_DECL;
    auto row_time = [&](int r) -> long long { return a.row_t ? (long long)a.row_t[r] : (long long)a.t0 + r; };

    if (warp == 0) {
        if (lane == 0) {
            // ------------------------------------------------------------ TMA producer (both CTAs)
            int stage = 0;
            uint32_t phase = 0;
            for (int it = 0; it < niter; ++it) {
                int mt, nt;
                unit_tile(it, mt, nt);
                if (RESB) {  // this unit's weight half, once
                    if (it > 0) mbar_wait(bempty_bar, (uint32_t)(it - 1) & 1u);
                    if (rank == 0) mbar_expect_tx(bfull_bar, 2u * a.num_kb * Cfg::B_BYTES);
                    for (int kb = 0; kb < a.num_kb; ++kb)
                        tma_load_2d_2sm(bres + kb * Cfg::B_BYTES, &tb, bfull_bar, kb * CL_BK, nt * BN + rank * (BN / 2));
                }
                for (int r = r_mma0; r < a.R; ++r) {
                    const long long m0 = (long long)row_of(r) * BHW + (long long)mt * CL_BM;  // flat input pixel
                    const int n0 = (int)(m0 / HW);
                    const int y0 = (int)((m0 % HW) / a.W);
                    for (int kb = 0; kb < steps; ++kb) {
                        const int tap = kb / a.conv_cb, cblk = kb % a.conv_cb;
                        CL_T0;
                        mbar_wait(empty_bar(stage), phase ^ 1u);
                        CL_T1(1);
                        const uint32_t sa = sring + stage * SBYTES;
                        const uint32_t fb = full_bar(stage);
                        if (a.diag & 16) {  // diagnostic: no loads (MMA on stale smem)
                            if (!PAIR || rank == 0) mbar_arrive(fb);
                        } else if (HALO) {  // step = (cblk, dx): halo box + weights of taps (dy, dx), dy = -1..1
                            const int hc = kb / 3, dxi = kb % 3;
                            const uint32_t bytes = a.halo_bytes + (RESB ? 0u : 3u * Cfg::B_BYTES);
                            if (PAIR) {
                                if (rank == 0) mbar_expect_tx(fb, 2 * bytes);
                                tma_load_4d_2sm(sa, &ta, fb, hc * CL_BK, dxi - 1, y0 - 1, n0);
                            } else {
                                mbar_expect_tx(fb, bytes);
                                tma_load_4d(sa, &ta, fb, hc * CL_BK, dxi - 1, y0 - 1, n0);
                            }
                            if (!RESB) {
#pragma unroll
                                for (int dyi = 0; dyi < 3; ++dyi) {
                                    const int kc = (wtap(dyi * 3 + dxi) * a.conv_cb + hc) * CL_BK;
                                    if (PAIR)
                                        tma_load_2d_2sm(sa + CL_AH_MAX + dyi * Cfg::B_BYTES, &tb, fb, kc,
                                                        nt * BN + rank * (BN / 2));
                                    else
                                        tma_load_2d(sa + CL_AH_MAX + dyi * Cfg::B_BYTES, &tb, fb, kc, nt * BN);
                                }
                            }
                        } else if (PAIR) {
                            // both CTAs' bytes land on the leader's full barrier
                            if (rank == 0) mbar_expect_tx(fb, 2 * SBYTES);
                            tma_load_4d_2sm(sa, &ta, fb, cblk * CL_BK, tap % 3 - 1, y0 + tap / 3 - 1, n0);
                            if (!RESB)
                                tma_load_2d_2sm(sa + Cfg::A_BYTES, &tb, fb, (wtap(tap) * a.conv_cb + cblk) * CL_BK,
                                                nt * BN + rank * (BN / 2));
                        } else {
                            mbar_expect_tx(fb, Cfg::STAGE_BYTES);
                            if (a.diag & 8)  // diagnostic: A as a 2D box of the flat [pixels][cin] view
                                tma_load_2d(sa, &ta, fb, cblk * CL_BK, (int)m0);
                            else if (a.diag & 4)  // diagnostic: centre tap only (no out-of-bounds lines)
                                tma_load_4d(sa, &ta, fb, cblk * CL_BK, 0, y0, n0);
                            else
                                tma_load_4d(sa, &ta, fb, cblk * CL_BK, tap % 3 - 1, y0 + tap / 3 - 1, n0);
                            tma_load_2d(sa + Cfg::A_BYTES, &tb, fb, (wtap(tap) * a.conv_cb + cblk) * CL_BK, nt * BN);
                        }
                        if (++stage == STAGES) {
                            stage = 0;
                            phase ^= 1u;
                        }
                    }
                }
            }
        }
    } else if (warp == 1) {
        if (lane == 0 && rank == 0) {
            // ------------------------------------------------------------ MMA issuer (leader)
            constexpr uint32_t idesc = umma_idesc_bf16(PAIR ? 2 * CL_BM : CL_BM, BN, 0, 0);
            int stage = 0;
            uint32_t phase = 0;
            int acc = 0;
            uint32_t acc_phase = 0;
            for (int it = 0; it < niter; ++it) {
                if (RESB) {
                    mbar_wait(bfull_bar, (uint32_t)it & 1u);
                    tc_fence_after();
                }
                for (int r = r_mma0; r < a.R; ++r) {
                    CL_T0;
                    mbar_wait(tempty_bar(acc), acc_phase ^ 1u);
                    CL_T1(1);
                    tc_fence_after();
                    const uint32_t d_tmem = tmem_base + acc * BN;
                    for (int kb = 0; kb < steps; ++kb) {
                        CL_T0;
                        mbar_wait(full_bar(stage), phase);
                        CL_T1(2);
                        tc_fence_after();
                        const uint32_t sa = sring + stage * SBYTES;
                        const uint32_t sb = RESB ? bres + kb * Cfg::B_BYTES : sa + A_STAGE;
#pragma unroll
                        for (int dyi = 0; dyi < (HALO ? 3 : 1); ++dyi) {
                            const uint32_t sad = sa + (uint32_t)dyi * (uint32_t)a.W * 128u;  // dy shift: W rows
                            uint32_t sbd = sb + (uint32_t)dyi * Cfg::B_BYTES;
                            if (HALO && RESB)  // resident weights of tap (dy, dx) for this channel block
                                sbd = bres + (uint32_t)(((dyi * 3 + kb % 3) * a.conv_cb + kb / 3) * Cfg::B_BYTES);
#pragma unroll
                            for (int k = 0; k < CL_BK / 16; ++k) {
                                if (a.diag & 2) break;  // diagnostic: no MMA
                                const uint64_t ad = umma_desc_sw128(sad + k * 32u, 16u, 1024u);
                                const uint64_t bd = umma_desc_sw128(sbd + k * 32u, 16u, 1024u);
                                const uint32_t accum = (kb > 0 || dyi > 0 || k > 0) ? 1u : 0u;
                                if (PAIR)
                                    tc_mma_f16_2sm(d_tmem, ad, bd, idesc, accum);
                                else
                                    tc_mma_f16(d_tmem, ad, bd, idesc, accum);
                            }
                        }
                        if (PAIR)
                            tc_commit_2sm_mc(empty_bar(stage), 3);
                        else
                            tc_commit(empty_bar(stage));
                        if (++stage == STAGES) {
                            stage = 0;
                            phase ^= 1u;
                        }
                    }
                    if (PAIR)
                        tc_commit_2sm_mc(tfull_bar(acc), 3);
                    else
                        tc_commit(tfull_bar(acc));
                    if (++acc == NACC) {
                        acc = 0;
                        acc_phase ^= 1u;
                    }
                }
                if (RESB) tc_commit_2sm_mc(bempty_bar, 3);  // this unit's weights may be replaced
            }
        }
    } else if constexpr (BWD != 0) {
        // ---------------------------------------------------------------- epilogue: reverse scan (Eq.2)
        // thread = pixel p of the tile, CW channels; delta of the unit in registers across the rows (the
        // carry), U of the next row prefetched while this row's accumulator is awaited
        const int q = warp & 3;
        const int h = (warp - 2) >> 2;
        const int p = q * 32 + lane;
        const long long rs = (long long)BHW * a.Cout;  // neurons per row
        const float th = a.theta, inv_th = 1.0f / a.theta, lam = a.lam, gam = a.gamma;
        auto sgm = [&](float u) -> float {  // sigma'(u), reading 4 (as lif_bwd_kernel with gs = 1)
            if (BWD == 1) return gam * fmaxf(0.0f, 1.0f - fabsf(u - th) * inv_th);
            const float dd = 1.0f + gam * fabsf(u - th);
            return __frcp_rn(dd * dd);
        };
        int acc = 0;
        uint32_t acc_phase = 0;
        for (int it = 0; it < niter; ++it) {
            int mt, nt;
            const bool uvalid = unit_tile(it, mt, nt);
            const int pg = mt * CL_BM + p;
            const bool valid = uvalid && pg < BHW;
            const int ch0 = nt * BN + h * CW;
            const long long nidx = (long long)(valid ? pg : 0) * a.Cout + ch0;
            float d[CW];
            auto load8 = [&](const float *src, float *dst) {
                uint4 x0, x1;
                ldg_v8u(src, x0, x1);
                dst[0] = __uint_as_float(x0.x); dst[1] = __uint_as_float(x0.y); dst[2] = __uint_as_float(x0.z);
                dst[3] = __uint_as_float(x0.w); dst[4] = __uint_as_float(x1.x); dst[5] = __uint_as_float(x1.y);
                dst[6] = __uint_as_float(x1.z); dst[7] = __uint_as_float(x1.w);
            };
#pragma unroll
            for (int c = 0; c < CW; ++c) d[c] = 0.f;
            if (valid) {
#pragma unroll
                for (int c = 0; c < CW; c += 8) load8(a.bcarry + nidx + c, d + c);
            }
            for (int r = 0; r < a.R; ++r) {
                const int rr = a.R - 1 - r;
                const float *Ur = a.bU + (long long)rr * rs + nidx;
                // U of this row, 32 channels at a time: chunk 0 is requested before the accumulator wait
                float u[32];
#pragma unroll
                for (int c = 0; c < 32; ++c) u[c] = 0.f;
                if (valid) {
#pragma unroll
                    for (int c = 0; c < 32; c += 8) load8(Ur + c, u + c);
                }
                mbar_wait(tfull_bar(acc), acc_phase);
                tc_fence_after();
#pragma unroll
                for (int j = 0; j < CW / 32; ++j) {
                    if (j > 0 && valid) {
#pragma unroll
                        for (int c = 0; c < 32; c += 8) load8(Ur + 32 * j + c, u + c);
                    }
                    uint32_t v[32];
                    tmem_ld_32x32b_x32(tmem_base + ((uint32_t)(q * 32) << 16) + acc * BN + h * CW + j * 32, v);
                    tmem_ld_wait();
#pragma unroll
                    for (int c = 0; c < 32; ++c)
                        d[32 * j + c] = sgm(u[c]) * __uint_as_float(v[c]) + lam * d[32 * j + c];  // as lif_bwd_kernel
                }
                tc_fence_before();
                __syncwarp();
                if (lane == 0) {
                    if (PAIR)
                        mbar_arrive_leader(tempty_bar(acc));
                    else
                        mbar_arrive(tempty_bar(acc));
                }
                if (++acc == NACC) {
                    acc = 0;
                    acc_phase ^= 1u;
                }
                if (valid) {  // bf16 delta, 16 channels (one 32-byte sector) per store
                    uint16_t *dst = a.bdelta + (long long)rr * rs + nidx;
#pragma unroll
                    for (int c = 0; c < CW; c += 16) {
                        uint32_t pk[8];
#pragma unroll
                        for (int e = 0; e < 8; ++e)
                            pk[e] = (uint32_t)f2bf_bits(d[c + 2 * e]) | ((uint32_t)f2bf_bits(d[c + 2 * e + 1]) << 16);
                        st_global_v8u(dst + c, make_uint4(pk[0], pk[1], pk[2], pk[3]), make_uint4(pk[4], pk[5], pk[6], pk[7]));
                    }
                }
            }
            if (valid) {
#pragma unroll
                for (int c = 0; c < CW; c += 8) st_global_v8(a.bcarry + nidx + c, d + c);
            }
        }
    } else {
        // ---------------------------------------------------------------- epilogue: LIF over rows
        const int q = warp & 3;
        const int h = (warp - 2) >> 2;
        const int p = q * 32 + lane;  // tile row = output pixel
        const int etid = threadIdx.x - 64;  // 0..255
        const long long rs = (long long)BHW * a.Cout;  // neurons per row
        const int PH = a.H / 2, PW = a.W / 2;
        const long long prs = POOL ? rs / 4 : rs;  // outputs per row
        // tile geometry: rows of W pixels, bh image rows per image, 128 / (bh * W) images
        const int bh = HW >= CL_BM ? CL_BM / a.W : a.H;
        int acc = 0;
        uint32_t acc_phase = 0;
        uint32_t ebuf = 0;  // spike exchange buffer parity, flips every emitted row (across units too)
        for (int it = 0; it < niter; ++it) {
            int mt, nt;
            const bool uvalid = unit_tile(it, mt, nt);
            const int pg = mt * CL_BM + p;  // pixel within a row
            const bool valid = uvalid && pg < BHW;
            const int ch0 = nt * BN + h * CW;
            const long long nidx = (long long)(valid ? pg : 0) * a.Cout + ch0;
            // state / checkpoint element of channel c (multiple of 4): NHWC, or thread-major (a.state_tm:
            // [unit][half][c/4][pixel of the tile][4], so a warp's float4 / uchar4 accesses are contiguous)
            const long long tm0 = ((((long long)mt * a.n_tiles + nt) * 2 + h) * (CW / 4) * CL_BM + p) * 4;
            auto sidx = [&](int c) -> long long { return a.state_tm ? tm0 + (long long)(c >> 2) * (CL_BM * 4) : nidx + c; };
            float U[CW];
            uint32_t ob[CW / 32];
            if (valid && !(a.diag & 32)) {  // diag 32: no state load / store (timing experiment)
#pragma unroll
                for (int c = 0; c < CW; c += 4) {
                    const float4 v = *reinterpret_cast<const float4 *>(a.U_state + sidx(c));
                    U[c] = v.x; U[c + 1] = v.y; U[c + 2] = v.z; U[c + 3] = v.w;
                }
#pragma unroll
                for (int j = 0; j < CW / 32; ++j) {
                    uint32_t w = 0;
#pragma unroll
                    for (int c = 0; c < 32; c += 4) {
                        const uchar4 o4 = *reinterpret_cast<const uchar4 *>(a.o_state + sidx(32 * j + c));
                        w |= (o4.x ? 1u : 0u) << c | (o4.y ? 1u : 0u) << (c + 1) | (o4.z ? 1u : 0u) << (c + 2) |
                             (o4.w ? 1u : 0u) << (c + 3);
                    }
                    ob[j] = w;
                }
            } else {
#pragma unroll
                for (int c = 0; c < CW; ++c) U[c] = 0.f;
#pragma unroll
                for (int j = 0; j < CW / 32; ++j) ob[j] = 0u;
            }
            // state-layout stores (running state, checkpoint) when tm, else NHWC at nidx (debug record)
            auto store_state = [&](float *Ud, uint8_t *od, bool tm) {
#pragma unroll
                for (int c = 0; c < CW; c += 4) {
                    const long long e = tm ? sidx(c) : nidx + c;
                    *reinterpret_cast<float4 *>(Ud + e) = make_float4(U[c], U[c + 1], U[c + 2], U[c + 3]);
                    const uint32_t w = ob[c >> 5] >> (c & 31);
                    *reinterpret_cast<uchar4 *>(od + e) = make_uchar4(w & 1u, (w >> 1) & 1u, (w >> 2) & 1u, (w >> 3) & 1u);
                }
            };
            auto emit = [&](int r) {
                const long long t = row_time(r);
                unsigned cnt = 0;
                if (a.u2_part) {  // l2-trace SAM (reading 25): this thread's U^2, summed per warp
                    double q2 = 0.0;
                    if (valid) {
#pragma unroll
                        for (int c = 0; c < CW; ++c) q2 += (double)U[c] * (double)U[c];
                    }
                    u2_warp_add(a.u2_part, t, q2);
                }
                if (valid) {
#pragma unroll
                    for (int j = 0; j < CW / 32; ++j) cnt += __popc(ob[j]);
                    if (a.U_out) {
                        float *dst = a.U_out + (long long)r * rs + nidx;
#pragma unroll
                        for (int c = 0; c < CW; c += 8) st_global_v8(dst + c, U + c);
                    }
                    if (a.dbg_U) store_state(a.dbg_U + t * rs, a.dbg_o + t * rs, false);
                    if (!POOL) {  // bf16 spikes, 16 channels (one 32-byte sector) per store
                        uint16_t *dst = a.Po_out + (long long)r * rs + nidx;
#pragma unroll
                        for (int c = 0; c < CW; c += 16) {
                            const uint32_t w = ob[c >> 5] >> (c & 31);
                            uint32_t pk[8];
#pragma unroll
                            for (int e = 0; e < 8; ++e)
                                pk[e] = (((w >> (2 * e)) & 1u) ? 0x3F80u : 0u) | (((w >> (2 * e + 1)) & 1u) ? 0x3F800000u : 0u);
                            st_global_v8u(dst + c, make_uint4(pk[0], pk[1], pk[2], pk[3]), make_uint4(pk[4], pk[5], pk[6], pk[7]));
                        }
                    }
                }
                if (POOL) {
                    // spike words -> smem [pixel][word] (buffer r & 1), then 2x2 window sums by all
                    // epilogue threads: item = (pooled pixel of the tile, 8-channel group)
                    uint32_t *sw = s_spk + (ebuf & 1u) * (CL_BM * NW);
                    ++ebuf;
#pragma unroll
                    for (int j = 0; j < CW / 32; ++j) sw[p * NW + h * (CW / 32) + j] = valid ? ob[j] : 0u;
                    asm volatile("bar.sync 1, %0;" ::"n"(32 * CL_EPI_WARPS) : "memory");
                    const int PWt = a.W / 2, PHt = bh / 2;
                    constexpr int GROUPS = BN / 8;
                    for (int it = etid; it < (CL_BM / 4) * GROUPS; it += 32 * CL_EPI_WARPS) {
                        const int qp = it / GROUPS, gsel = it % GROUPS;
                        const int img = qp / (PHt * PWt), py = (qp / PWt) % PHt, px = qp % PWt;
                        const int p00 = (img * bh + 2 * py) * a.W + 2 * px;
                        const int pg00 = mt * CL_BM + p00;
                        if (!uvalid || pg00 >= BHW) continue;
                        const int wsel = gsel >> 2, sh = (gsel & 3) * 8;
                        const uint32_t w0 = sw[p00 * NW + wsel] >> sh, w1 = sw[(p00 + 1) * NW + wsel] >> sh;
                        const uint32_t w2 = sw[(p00 + a.W) * NW + wsel] >> sh, w3 = sw[(p00 + a.W + 1) * NW + wsel] >> sh;
                        uint32_t pk[4];
#pragma unroll
                        for (int e = 0; e < 4; ++e) {
                            uint32_t v2 = 0;
#pragma unroll
                            for (int hh = 0; hh < 2; ++hh) {
                                const int ch = 2 * e + hh;
                                const uint32_t n = ((w0 >> ch) & 1u) + ((w1 >> ch) & 1u) + ((w2 >> ch) & 1u) + ((w3 >> ch) & 1u);
                                v2 |= (__float_as_uint(__uint2float_rn(n) * 0.25f) >> 16) << (16 * hh);
                            }
                            pk[e] = v2;
                        }
                        const int b = pg00 / HW, yy = (pg00 % HW) / a.W, xx = pg00 % a.W;
                        const long long oidx = (((long long)b * PH + (yy >> 1)) * PW + (xx >> 1)) * a.Cout + nt * BN + gsel * 8;
                        *reinterpret_cast<uint4 *>(a.Po_out + (long long)r * prs + oidx) = make_uint4(pk[0], pk[1], pk[2], pk[3]);
                    }
                }
                if (a.s_part) {
                    const unsigned v = __reduce_add_sync(0xffffffffu, cnt);
                    if (lane == 0 && v) atomicAdd(&s_cnt[r], v);
                }
            };

            if (a.restore && !(a.diag & 1)) emit(0);
            CkCursor ck(r_mma0, a.ck_every);
            for (int r = r_mma0; r < a.R; ++r) {
                CL_T0;
                mbar_wait_sleep(tfull_bar(acc), acc_phase);
                CL_T1(1);
                CL_T0;
                tc_fence_after();
#pragma unroll
                for (int j = 0; j < CW / 32; ++j) {
                    if (a.diag & 1) break;  // diagnostic: epilogue does no LIF / output work
                    uint32_t v[32];
                    tmem_ld_32x32b_x32(tmem_base + ((uint32_t)(q * 32) << 16) + acc * BN + h * CW + j * 32, v);
                    tmem_ld_wait();
                    uint32_t nb = 0;
#pragma unroll
                    for (int c = 0; c < 32; ++c) {
                        const float uu = cl_lif(U[32 * j + c], __uint_as_float(v[c]), (float)((ob[j] >> c) & 1u), a.lam, a.theta);
                        U[32 * j + c] = uu;
                        nb |= (uu > a.theta ? 1u : 0u) << c;
                    }
                    ob[j] = nb;
                }
                tc_fence_before();
                __syncwarp();
                if (lane == 0) {
                    if (PAIR)
                        mbar_arrive_leader(tempty_bar(acc));
                    else
                        mbar_arrive(tempty_bar(acc));
                }
                if (++acc == NACC) {
                    acc = 0;
                    acc_phase ^= 1u;
                }
                CL_T1(2);
                CL_T0;
                if (!(a.diag & 1)) emit(r);
                CL_T1(3);
                int ck_slot;
                if (ck.hit(r, ck_slot) && a.ckU && valid) {
                    const long long slot = (long long)ck_slot * a.ck_stride;
                    store_state(a.ckU + slot, a.cko + slot, true);
                }
            }
            if (!a.restore && valid && !(a.diag & 32)) store_state(a.U_state, a.o_state, true);
        }
    }
    tc_fence_before();
    __syncthreads();
    if (PAIR) cluster_sync_all();  // no CTA leaves while its peer may still signal its barriers
    tc_fence_after();
    if (warp == 1) {
        if (PAIR)
            tmem_dealloc_2sm<Cfg::TMEM_COLS>(tmem_base);
        else
            tmem_dealloc<Cfg::TMEM_COLS>(tmem_base);
    }
    CL_STAT_DUMP;
    if (a.s_part) {
        for (int r = threadIdx.x; r < a.R; r += blockDim.x) {
            const unsigned v = s_cnt[r];
            if (v) atomicAdd(a.s_part + row_time(r) * 32 + (blockIdx.x & 31), v);
        }
    }
}

long long conv_lif_state_count(int B, int H, int W, int cout) {
    return ((long long)B * H * W + CL_BM - 1) / CL_BM * CL_BM * cout;
}

bool conv_lif_supported(int B, int H, int W, int cin, int cout, int pool) {
    if (cin % 64 || (cout != 64 && cout % 128)) return false;
    if (W > CL_BM || CL_BM % W) return false;
    const int HW = H * W;
    if (HW >= CL_BM) {
        const int bh = CL_BM / W;
        if (H % bh) return false;
        if (pool && bh % 2) return false;
    } else if (CL_BM % HW) {
        return false;
    }
    if (pool && (H % 2 || W % 2)) return false;
    (void)B;
    return true;
}

template <int BN, int POOL, int PAIR, int RESB, int HALO, int BWD = 0>
static cudaError_t launch_cl(const CUtensorMap &ta, const CUtensorMap &tb, ConvLifArgs a, cudaStream_t s,
                             int num_sms) {
    using Cfg = ClCfg<BN, PAIR>;
    auto kern = conv_lif_kernel<BN, POOL, PAIR, RESB, HALO, BWD>;
    uint32_t smem = Cfg::FIXED_BYTES + 4u * (uint32_t)a.R + 16;
    const uint32_t resb = RESB ? (uint32_t)a.num_kb * Cfg::B_BYTES : 0u;
    const uint32_t sbytes = (HALO ? CL_AH_MAX : Cfg::A_BYTES) + (RESB ? 0u : (HALO ? 3u : 1u) * Cfg::B_BYTES);
    const int room = (int)((227u * 1024u - smem - resb) / sbytes);
    a.stages = room < CL_MAXST ? room : CL_MAXST;
    if (a.stages < 2) return cudaErrorInvalidValue;
    smem += resb + a.stages * sbytes;
    if (smem > 227u * 1024u) return cudaErrorInvalidValue;
    static uint32_t set = 0;
    if (smem > set) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        set = smem;
    }
    const int workers = PAIR ? (a.m_tiles / 2) * a.n_tiles : a.m_tiles * a.n_tiles;
    const int max_workers = PAIR ? num_sms / 2 : num_sms;
    const int grid = (workers < max_workers ? workers : max_workers) * (PAIR ? 2 : 1);
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(CL_THREADS);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute attrs[2];
    attrs[0].id = cudaLaunchAttributeClusterDimension;
    attrs[0].val.clusterDim.x = PAIR ? 2 : 1;
    attrs[0].val.clusterDim.y = 1;
    attrs[0].val.clusterDim.z = 1;
    attrs[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attrs[1].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
    cfg.attrs = attrs;
    cfg.numAttrs = 2;
    return cudaLaunchKernelEx(&cfg, kern, ta, tb, a);
}

// CTA pairs (SKIPPER_CL_PAIR=0 disables) when the pixel tiles of a channel tile pair up
static bool cl_use_pair(int m_tiles) {
    const char *e = getenv("SKIPPER_CL_PAIR");  // read per launch so tests can cover both variants
    // default on since the halo boxes and PDL: pairs measured ~0.4-0.7 % faster per step on cfg 2 and
    // cfg 3 (alternating repetitions); before the halo boxes they were ~2 % slower.  The kernel stays
    // bound by its TMA producer skeleton either way.
    return (!e || atoi(e) != 0) && m_tiles % 2 == 0;
}

cudaError_t launch_conv_lif(const void *X, int rows_in, const void *Wk, ConvLifArgs a, cudaStream_t s, int num_sms) {
    if (!conv_lif_supported(a.B, a.H, a.W, a.Cin, a.Cout, a.pool)) return cudaErrorInvalidValue;
    if (a.R <= 0) return cudaSuccess;
    const int bn = a.Cout == 64 ? 64 : 128;
    const int HW = a.H * a.W;
    uint32_t bw = a.W, bhh, bnn;
    if (HW >= CL_BM) {
        bhh = CL_BM / a.W;
        bnn = 1;
    } else {
        bhh = a.H;
        bnn = CL_BM / HW;
    }
    a.conv_cb = a.Cin / 64;
    a.num_kb = 9 * a.conv_cb;
    a.m_tiles = (a.B * HW + CL_BM - 1) / CL_BM;
    a.n_tiles = a.Cout / bn;
    const bool pair = cl_use_pair(a.m_tiles);
    {
        static const int diag = getenv("SKIPPER_CL_DIAG") ? atoi(getenv("SKIPPER_CL_DIAG")) : 0;
        a.diag = diag;  // timing experiments only (results are wrong when set)
    }

    CUtensorMap ta, tb;
    // halo boxes: single CTA, tiles of whole image rows of one image, W >= 8 (dy offsets of W rows
    // stay on 1024-byte swizzle atoms), box within CL_AH_MAX
    const char *he = getenv("SKIPPER_CL_HALO");
    const bool halo = !(he && atoi(he) == 0) && HW >= CL_BM && a.W >= 8 && a.W <= 32 && !(a.diag & 12);
    a.halo_bytes = halo ? (int)((bhh + 2) * bw * 128u) : 0;
    if (a.diag & 8) {
        if (!make_map_2d(&ta, X, a.Cin, (uint64_t)rows_in * a.B * HW, CL_BK, CL_BM)) return cudaErrorInvalidValue;
    } else if (!make_map_conv(&ta, X, a.Cin, a.W, a.H, (uint64_t)rows_in * a.B, bw, halo ? bhh + 2 : bhh, bnn)) {
        return cudaErrorInvalidValue;
    }
    if (!make_map_2d(&tb, Wk, 9ull * a.Cin, a.Cout, CL_BK, pair ? bn / 2 : bn)) return cudaErrorInvalidValue;
    // resident weights when this CTA's half fits next to >= 4 activation stages
    // resident weight halves: opt-in (SKIPPER_CL_RESB=1); streaming them measured ~0.3 % faster per step on
    // cfg 2 and cfg 3 (alternating repetitions): the resident halves leave room for only ~one row of
    // activation stages
    const int resb_env = getenv("SKIPPER_CL_RESB") ? atoi(getenv("SKIPPER_CL_RESB")) : 0;
    const uint32_t half_bytes = (uint32_t)a.num_kb * (uint32_t)(bn / 2) * CL_BK * 2;
    const bool resb = pair && resb_env && half_bytes + 3u * CL_AH_MAX + 8192u + 4u * a.R <= 226u * 1024u;
#define CL_LAUNCH(BN_, PAIR_, RESB_, HALO_)                                                                    \
    return a.pool ? launch_cl<BN_, 1, PAIR_, RESB_, HALO_>(ta, tb, a, s, num_sms)                               \
                  : launch_cl<BN_, 0, PAIR_, RESB_, HALO_>(ta, tb, a, s, num_sms)
    if (bn == 64) {
        if (resb && halo) CL_LAUNCH(64, 1, 1, 1);
        if (resb) CL_LAUNCH(64, 1, 1, 0);
        if (pair && halo) CL_LAUNCH(64, 1, 0, 1);
        if (pair) CL_LAUNCH(64, 1, 0, 0);
        if (halo) CL_LAUNCH(64, 0, 0, 1);
        CL_LAUNCH(64, 0, 0, 0);
    }
    if (resb && halo) CL_LAUNCH(128, 1, 1, 1);
    if (resb) CL_LAUNCH(128, 1, 1, 0);
    if (pair && halo) CL_LAUNCH(128, 1, 0, 1);
    if (pair) CL_LAUNCH(128, 1, 0, 0);
    if (halo) CL_LAUNCH(128, 0, 0, 1);
    CL_LAUNCH(128, 0, 0, 0);
#undef CL_LAUNCH
}

bool conv_lif_bwd_supported(int B, int H, int W, int cin, int cout) {
    return cout % 64 == 0 && conv_lif_supported(B, H, W, cin, cout, 0);
}

cudaError_t launch_conv_lif_bwd(const void *D, int rows_in, const void *Wt, ConvLifArgs a, cudaStream_t s, int num_sms) {
    if (!conv_lif_bwd_supported(a.B, a.H, a.W, a.Cin, a.Cout) || !a.bU || !a.bcarry || !a.bdelta)
        return cudaErrorInvalidValue;
    if (a.R <= 0) return cudaSuccess;
    if (rows_in < a.R) return cudaErrorInvalidValue;
    // 128-channel tiles (64 channels per epilogue thread: carry + one 32-channel U chunk + accumulator chunk
    // in registers) halve the activation ingress per MMA against 64-channel tiles (SKIPPER_CLB_BN64=1)
    const char *e64 = getenv("SKIPPER_CLB_BN64");
    const int bn = (a.Cout % 128 == 0 && !(e64 && atoi(e64))) ? 128 : 64;
    const int HW = a.H * a.W;
    uint32_t bhh, bnn;
    if (HW >= CL_BM) {
        bhh = CL_BM / a.W;
        bnn = 1;
    } else {
        bhh = a.H;
        bnn = CL_BM / HW;
    }
    a.pool = 0;
    a.restore = 0;
    a.conv_cb = a.Cin / 64;
    a.num_kb = 9 * a.conv_cb;
    a.m_tiles = (a.B * HW + CL_BM - 1) / CL_BM;
    a.n_tiles = a.Cout / bn;
    a.diag = 0;
    const bool pair = cl_use_pair(a.m_tiles);
    const char *he = getenv("SKIPPER_CL_HALO");
    const bool halo = !(he && atoi(he) == 0) && HW >= CL_BM && a.W >= 8 && a.W <= 32;
    a.halo_bytes = halo ? (int)((bhh + 2) * (uint32_t)a.W * 128u) : 0;
    CUtensorMap ta, tb;
    if (!make_map_conv(&ta, D, a.Cin, a.W, a.H, (uint64_t)rows_in * a.B, a.W, halo ? bhh + 2 : bhh, bnn))
        return cudaErrorInvalidValue;
    if (!make_map_2d(&tb, Wt, 9ull * a.Cin, a.Cout, CL_BK, pair ? bn / 2 : bn)) return cudaErrorInvalidValue;
    const bool tri = a.surr == 0;
#define CLB_LAUNCH(BN_, PAIR_, HALO_)                                          \
    return tri ? launch_cl<BN_, 0, PAIR_, 0, HALO_, 1>(ta, tb, a, s, num_sms) \
               : launch_cl<BN_, 0, PAIR_, 0, HALO_, 2>(ta, tb, a, s, num_sms)
    if (bn == 128) {
        if (pair && halo) CLB_LAUNCH(128, 1, 1);
        if (pair) CLB_LAUNCH(128, 1, 0);
        if (halo) CLB_LAUNCH(128, 0, 1);
        CLB_LAUNCH(128, 0, 0);
    }
    if (pair && halo) CLB_LAUNCH(64, 1, 1);
    if (pair) CLB_LAUNCH(64, 1, 0);
    if (halo) CLB_LAUNCH(64, 0, 1);
    CLB_LAUNCH(64, 0, 0);
#undef CLB_LAUNCH
}

}  // namespace sk
