// gemm_tc.cu - K2: synaptic contractions on the 5th-generation tensor cores (sm_100a).
//
// One persistent, warp-specialised kernel family:
//   warp 0      TMA producer  (cp.async.bulk.tensor -> 128B-swizzled smem ring, mbarrier complete_tx)
//   warp 1      MMA issuer    (one thread: tcgen05.mma.cta_group::1.kind::f16, M=128, N=BN, K=16,
//                              accumulators in TMEM, tcgen05.commit frees smem stages)
//               + TMEM allocator (2 accumulator buffers so the epilogue of tile i overlaps tile i+1)
//   warps 2-5   epilogue      (tcgen05.ld 32x32b -> registers -> 128B-swizzled smem -> TMA store, or
//                              TMA reduce-add for split-K weight gradients)
// Operands are bf16 (exact for spikes and grid weights), accumulation fp32.
// Convolutions are implicit GEMMs: each K block is one 3x3 tap x 64 channels, loaded by a 4D TMA
// box shifted by the tap offset; the zero padding is TMA's out-of-bounds fill.
#include "common.cuh"
#include "gemm.h"

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <mutex>

namespace sk {

static constexpr int BM = 128;
static constexpr int BK = 64;        // bf16 elements per K block = one 128-byte swizzle row
static constexpr int NUM_THREADS = 192;
// MN-major (weight-gradient) kernels carry a 7th warp that zero-fixes OP_MNSHIFT operand rows
template <int MN>
static constexpr int kThreads = MN ? 224 : 192;

template <int BN>
struct GemmCfg {
    static constexpr uint32_t A_BYTES = BM * BK * 2;
    static constexpr uint32_t B_BYTES = BN * BK * 2;
    static constexpr uint32_t STAGE_BYTES = A_BYTES + B_BYTES;
    static constexpr int STAGES = (BN == 64) ? 8 : (BN == 128 ? 6 : 4);
    static constexpr uint32_t TMEM_COLS = (2 * BN <= 128) ? 128 : (2 * BN <= 256 ? 256 : 512);
    static constexpr uint32_t EPI_BYTES = 4 * 2 * 4096;  // 4 epilogue warps x 2 buffers x (32 x 32 fp32)
    static constexpr int MAX_RING = 48;  // narrow K blocks (plan_conv_s) run a deeper ring of smaller stages
    static constexpr uint32_t SMEM_BYTES = STAGES * STAGE_BYTES + EPI_BYTES + 1024 /*align*/ + 1024 /*barriers*/;
};

struct TileCoord {
    int m_t, n_t, tap, split, kb0, kb1;
};

// CS > 1: a cluster of CS CTAs walks groups of CS consecutive M tiles sharing one N tile; each CTA
// loads its own A tile and 1/CS of the B tile, multicast to the whole cluster.
template <int CS>
SK_DEV int iter_count(const GemmDev &g) {
    if (CS == 1) return g.m_tiles * g.n_tiles * g.taps * g.splits;
    return ((g.m_tiles + CS - 1) / CS) * g.n_tiles;
}

SK_DEV TileCoord decode_tile(const GemmDev &g, int tile);

template <int CS>
SK_DEV TileCoord tile_at(const GemmDev &g, int it, int rank) {
    if (CS == 1) return decode_tile(g, it);
    const int mg = (g.m_tiles + CS - 1) / CS;
    TileCoord c;
    c.m_t = (it % mg) * CS + rank;
    c.n_t = it / mg;
    c.tap = 0;
    c.split = 0;
    c.kb0 = 0;
    c.kb1 = g.num_kb;
    return c;
}

SK_DEV TileCoord decode_tile(const GemmDev &g, int tile) {
    TileCoord c;
    c.m_t = tile % g.m_tiles;
    int r = tile / g.m_tiles;
    c.n_t = r % g.n_tiles;
    r /= g.n_tiles;
    c.tap = r % g.taps;
    c.split = r / g.taps;
    c.kb0 = c.split * g.kb_per_split;
    c.kb1 = min(g.num_kb, c.kb0 + g.kb_per_split);
    return c;
}

// Optional pipeline statistics (g.stats != null): cycles each role spends blocked on its barrier.
SK_DEV void mbar_wait_t(uint32_t bar, uint32_t parity, unsigned long long *acc) {
    if (acc) {
        const long long t0 = clock64();
        mbar_wait(bar, parity);
        *acc += (unsigned long long)(clock64() - t0);
    } else {
        mbar_wait(bar, parity);
    }
}

template <int BN, int MN, int CS>
__global__ void __launch_bounds__(kThreads<MN>, 1)
    gemm_tc_kernel(const __grid_constant__ CUtensorMap ta, const __grid_constant__ CUtensorMap tb,
                   const __grid_constant__ CUtensorMap tcm, const GemmDev g) {
    pdl_enter();
    using Cfg = GemmCfg<BN>;
    constexpr int STAGES = Cfg::STAGES;
    extern __shared__ uint8_t smem_raw[];
    const uint32_t raw = smem_u32(smem_raw);
    const uint32_t base = (raw + 1023u) & ~1023u;
    const uint32_t epi = base + STAGES * Cfg::STAGE_BYTES;  // 1024-aligned (stage bytes are multiples of 1 KB)
    const uint32_t bars = epi + Cfg::EPI_BYTES;
    auto full_bar = [&](int s) { return bars + 8u * s; };
    constexpr int MR = Cfg::MAX_RING;
    auto empty_bar = [&](int s) { return bars + 8u * (MR + s); };
    auto tfull_bar = [&](int a) { return bars + 8u * (2 * MR + a); };
    auto tempty_bar = [&](int a) { return bars + 8u * (2 * MR + 2 + a); };
    const uint32_t tmem_slot = bars + 8u * (2 * MR + 4);
    auto fixed_bar = [&](int s) { return bars + 8u * (2 * MR + 6 + s); };  // OP_MNSHIFT: rows fixed (s < STAGES)
    // ring geometry: the compile-time stages, or (narrow K blocks) g.ring stages of g.stage_stride bytes
    const int nst = g.kblk ? g.ring : STAGES;
    const uint32_t sstride = g.kblk ? g.stage_stride : Cfg::STAGE_BYTES;
    const uint32_t a_bytes = g.kblk ? (uint32_t)BM * g.kblk * 2u : Cfg::A_BYTES;
    uint32_t *tmem_slot_ptr = reinterpret_cast<uint32_t *>(smem_raw + (tmem_slot - raw));

    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    unsigned long long w_stat = 0, *wst = g.stats ? &w_stat : nullptr;
    const long long t_start = clock64();

    if (warp == 0 && lane == 0) {
        tma_prefetch(&ta);
        tma_prefetch(&tb);
        tma_prefetch(&tcm);
        for (int s = 0; s < nst; ++s) {
            mbar_init(full_bar(s), 1);
            mbar_init(empty_bar(s), CS);  // every CTA of the cluster frees the stage (multicast B)
        }
        if (MN)
            for (int s = 0; s < STAGES; ++s) mbar_init(fixed_bar(s), 1);
        for (int a = 0; a < 2; ++a) {
            mbar_init(tfull_bar(a), 1);
            mbar_init(tempty_bar(a), 4);
        }
        fence_mbar_init();
    }
    if (warp == 1) tmem_alloc<Cfg::TMEM_COLS>(tmem_slot);
    tc_fence_before();
    if (CS > 1)
        cluster_sync_all();
    else
        __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *reinterpret_cast<volatile uint32_t *>(tmem_slot_ptr);

    const int total = iter_count<CS>(g);
    const int rank = CS > 1 ? (int)cluster_ctarank() : 0;
    const int it0 = CS > 1 ? (int)blockIdx.x / CS : (int)blockIdx.x;
    const int itstep = CS > 1 ? (int)gridDim.x / CS : (int)gridDim.x;
    constexpr uint16_t mc_mask = (uint16_t)((1u << CS) - 1u);

    if (warp == 0) {
        if (lane == 0) {
            // ------------------------------------------------------------ TMA producer
            int stage = 0;
            uint32_t phase = 0;
            for (int tile = it0; tile < total; tile += itstep) {
                const TileCoord tc = tile_at<CS>(g, tile, rank);
                const int tdy = tc.tap / 3 - 1, tdx = tc.tap % 3 - 1;
                for (int kb = tc.kb0; kb < tc.kb1; ++kb) {
                    mbar_wait_t(empty_bar(stage), phase ^ 1u, wst);
                    const uint32_t sa = base + stage * sstride;
                    const uint32_t sb = sa + a_bytes;
                    const uint32_t fb = full_bar(stage);
                    mbar_expect_tx(fb, g.kblk ? g.stage_tx : Cfg::STAGE_BYTES);
                    const int kbe = g.kblk ? g.kblk : BK;  // K elements per block
                    // ---- A
                    if (g.a_kind == OP_K2D) {
                        tma_load_2d(sa, &ta, fb, kb * BK, tc.m_t * BM);
                    } else if (g.a_kind == OP_KCONV) {
                        const int tap = kb / g.conv_cb, cblk = kb % g.conv_cb;
                        const int dy = tap / 3 - 1, dx = tap % 3 - 1;
                        const int m0 = tc.m_t * BM;
                        const int n0 = m0 / g.conv_hw;
                        const int y0 = (m0 % g.conv_hw) / g.conv_w;
                        if (g.kblk)  // strided / narrow: input rows s*y0 + dy, element strides in the map
                            tma_load_4d(sa, &ta, fb, cblk * kbe, g.conv_sign * dx,
                                        g.conv_stride * y0 + g.conv_sign * dy, n0);
                        else
                            tma_load_4d(sa, &ta, fb, cblk * BK, g.conv_sign * dx, y0 + g.conv_sign * dy, n0);
                    } else {  // OP_MN2D: two 64-wide MN chunks
                        tma_load_2d(sa, &ta, fb, tc.m_t * BM, kb * BK);
                        tma_load_2d(sa + 8192u, &ta, fb, tc.m_t * BM + 64, kb * BK);
                    }
                    // ---- B
                    if (CS > 1) {  // K-major B slice multicast to the cluster
                        constexpr uint32_t SL = BN / CS;
                        tma_load_2d_mc(sb + (uint32_t)rank * SL * 128u, &tb, fb, kb * BK, tc.n_t * BN + rank * (int)SL,
                                       mc_mask);
                    } else if (g.b_kind == OP_K2D) {
                        tma_load_2d(sb, &tb, fb, kb * kbe, tc.n_t * BN);
                    } else if (g.b_kind == OP_MN2D) {
#pragma unroll
                        for (int i = 0; i < BN / 64; ++i)
                            tma_load_2d(sb + 8192u * i, &tb, fb, tc.n_t * BN + 64 * i, kb * BK);
                    } else if (g.b_kind == OP_KCONV) {  // activations as the N operand (transposed conv)
                        const int tap = kb / g.conv_cb, cblk = kb % g.conv_cb;
                        const int dy = tap / 3 - 1, dx = tap % 3 - 1;
                        const int m0 = tc.n_t * BN;
                        const int n0 = m0 / g.conv_hw;
                        const int y0 = (m0 % g.conv_hw) / g.conv_w;
                        tma_load_4d(sb, &tb, fb, cblk * BK, g.conv_sign * dx, y0 + g.conv_sign * dy, n0);
                    } else if (g.b_kind == OP_MNSHIFT) {  // flattened pixels kb*64.. at the tap's row offset
#pragma unroll
                        for (int i = 0; i < BN / 64; ++i) {
                            int ci0 = tc.n_t * BN + 64 * i;
                            const int tp = ci0 / g.wg_cin;
                            ci0 -= tp * g.wg_cin;
                            tma_load_2d(sb + 8192u * i, &tb, fb, ci0, kb * BK + (tp / 3 - 1) * g.conv_w + (tp % 3 - 1));
                        }
                    } else {  // OP_MNCONV: K rows kb*64.. of the image, shifted by the tap of each 64-chunk
                        const int m0 = kb * BK;
                        const int n0 = m0 / g.conv_hw;
                        const int y0 = (m0 % g.conv_hw) / g.conv_w;
#pragma unroll
                        for (int i = 0; i < BN / 64; ++i) {
                            int ci0 = tc.n_t * BN + 64 * i, ddy = tdy, ddx = tdx;
                            if (g.wg_cin) {  // N = (tap, cin): this chunk's tap
                                const int tp = ci0 / g.wg_cin;
                                ci0 -= tp * g.wg_cin;
                                ddy = tp / 3 - 1;
                                ddx = tp % 3 - 1;
                            }
                            tma_load_4d(sb + 8192u * i, &tb, fb, ci0, ddx, y0 + ddy, n0);
                        }
                    }
                    if (++stage == nst) {
                        stage = 0;
                        phase ^= 1u;
                    }
                }
            }
        }
    } else if (warp == 1) {
        if (lane == 0) {
            // ------------------------------------------------------------ MMA issuer
            constexpr uint32_t idesc = umma_idesc_bf16(BM, BN, MN, MN);
            const bool fix = MN && g.b_kind == OP_MNSHIFT;  // stages pass through the fixer warp
            int stage = 0;
            uint32_t phase = 0;
            int acc = 0;
            uint32_t acc_phase = 0;
            for (int tile = it0; tile < total; tile += itstep) {
                const TileCoord tc = tile_at<CS>(g, tile, rank);
                mbar_wait_t(tempty_bar(acc), acc_phase ^ 1u, wst);
                tc_fence_after();
                const uint32_t d_tmem = tmem_base + acc * BN;
                for (int kb = tc.kb0; kb < tc.kb1; ++kb) {
                    const uint32_t rb = fix ? fixed_bar(stage) : full_bar(stage);
                    if (wst) {  // MMA waiting on TMA data is accounted separately (slot 4)
                        unsigned long long f = 0;
                        mbar_wait_t(rb, phase, &f);
                        atomicAdd(g.stats + 4, f);
                    } else {
                        mbar_wait(rb, phase);
                    }
                    tc_fence_after();
                    const uint32_t sa = base + stage * sstride;
                    const uint32_t sb = sa + a_bytes;
                    if (!MN && g.kblk) {  // narrow K block: 16/32 elements, 32B/64B swizzle atoms
                        const uint32_t rowb = (uint32_t)g.kblk * 2u, lay = g.kblk == 16 ? 6u : (g.kblk == 32 ? 4u : 2u);
                        for (int k = 0; k < g.kblk / 16; ++k) {
                            const uint64_t ad = umma_desc_kmajor(sa + k * 32u, 8u * rowb, lay);
                            const uint64_t bd = umma_desc_kmajor(sb + k * 32u, 8u * rowb, lay);
                            tc_mma_f16(d_tmem, ad, bd, idesc, (kb > tc.kb0 || k > 0) ? 1u : 0u);
                        }
                        tc_commit(empty_bar(stage));
                        if (++stage == nst) {
                            stage = 0;
                            phase ^= 1u;
                        }
                        continue;
                    }
#pragma unroll
                    for (int k = 0; k < BK / 16; ++k) {
                        uint64_t ad, bd;
                        if (MN) {
                            ad = umma_desc_sw128(sa + k * 2048u, 8192u, 1024u);
                            bd = umma_desc_sw128(sb + k * 2048u, 8192u, 1024u);
                        } else {
                            ad = umma_desc_sw128(sa + k * 32u, 16u, 1024u);
                            bd = umma_desc_sw128(sb + k * 32u, 16u, 1024u);
                        }
                        tc_mma_f16(d_tmem, ad, bd, idesc, (kb > tc.kb0 || k > 0) ? 1u : 0u);
                    }
                    if (CS > 1)
                        tc_commit_mc(empty_bar(stage), mc_mask);
                    else
                        tc_commit(empty_bar(stage));
                    if (++stage == nst) {
                        stage = 0;
                        phase ^= 1u;
                    }
                }
                tc_commit(tfull_bar(acc));
                acc ^= 1;
                if (acc == 0) acc_phase ^= 1u;
            }
        }
    } else if (MN && warp == 6) {
        // ------------------------------------------------------------ OP_MNSHIFT row fixer
        // B chunk i of a stage holds 64 channels of one tap (dy, dx) for the 64 flattened pixels of the
        // K block, loaded at row offset dy*W + dx: rows whose shifted pixel leaves its image hold a
        // neighbour's pixel and are zeroed here (conv zero padding) before the MMA reads the stage.
        if (g.b_kind == OP_MNSHIFT) {
            const int W = g.conv_w, H = g.conv_hw / g.conv_w;
            int stage = 0;
            uint32_t phase = 0;
            for (int tile = it0; tile < total; tile += itstep) {
                const TileCoord tc = tile_at<CS>(g, tile, rank);
                int dxs[BN / 64], dys[BN / 64];
#pragma unroll
                for (int i = 0; i < BN / 64; ++i) {
                    const int tp = (tc.n_t * BN + 64 * i) / g.wg_cin;
                    dys[i] = tp / 3 - 1;
                    dxs[i] = tp % 3 - 1;
                }
                for (int kb = tc.kb0; kb < tc.kb1; ++kb) {
                    mbar_wait(full_bar(stage), phase);
                    const uint32_t sb = base + stage * sstride + a_bytes;
                    // rows lane and lane + 32: a lane zeroes its own row of every chunk whose tap moves the pixel
                    // out of its image, 16-byte units in a lane-rotated order (the 8 lanes of a store phase hit
                    // 8 different bank groups although their rows are 128 B apart)
#pragma unroll
                    for (int h2 = 0; h2 < 2; ++h2) {
                        const int r = lane + 32 * h2;
                        const unsigned p = (unsigned)kb * BK + (unsigned)r;
                        const unsigned q = p / (unsigned)W;
                        const int x = (int)(p - q * (unsigned)W);
                        const int y = (int)(q % (unsigned)H);
#pragma unroll
                        for (int i = 0; i < BN / 64; ++i) {
                            const int xs = x + dxs[i], ys = y + dys[i];
                            if (xs < 0 || xs >= W || ys < 0 || ys >= H) {
                                const uint32_t row = sb + 8192u * i + 128u * (uint32_t)r;
#pragma unroll
                                for (int j = 0; j < 8; ++j)
                                    asm volatile("st.shared.v4.u32 [%0], {%1, %1, %1, %1};" ::"r"(row + 16u * (uint32_t)((j + lane) & 7)),
                                                 "r"(0u)
                                                 : "memory");
                            }
                        }
                    }
                    fence_async_shared();  // generic-proxy stores -> visible to the tensor core (async proxy)
                    __syncwarp();
                    if (lane == 0) mbar_arrive(fixed_bar(stage));
                    if (++stage == nst) {
                        stage = 0;
                        phase ^= 1u;
                    }
                }
            }
        }
    } else {
        // ---------------------------------------------------------------- epilogue
        // Each warp owns TMEM lanes [32q, 32q+32) = 32 output rows.  Per 32-column chunk: TMEM ->
        // registers -> a 4 KB smem box in the 128B-swizzle pattern (16-byte chunk j of row r at
        // position j ^ (r & 7): conflict-free) -> one TMA store (or reduce-add) per box; two boxes
        // per warp in flight.  TMA clips rows >= M and columns >= N.
        const int q = warp & 3;  // TMEM lane quadrant this warp may access
        const uint32_t ebuf0 = epi + (uint32_t)q * 8192u;
        int acc = 0;
        uint32_t acc_phase = 0;
        uint32_t nbox = 0;
        for (int tile = it0; tile < total; tile += itstep) {
            const TileCoord tc = tile_at<CS>(g, tile, rank);
            mbar_wait_t(tfull_bar(acc), acc_phase, lane == 0 ? wst : nullptr);
            tc_fence_after();
            const int row0 = tc.m_t * BM + q * 32;
#pragma unroll 1
            for (int c = 0; c < BN / 32; ++c) {
                uint32_t r[32];
                tmem_ld_32x32b_x32(tmem_base + ((uint32_t)(q * 32) << 16) + acc * BN + c * 32, r);
                tmem_ld_wait();
                const uint32_t buf = ebuf0 + (nbox & 1u) * 4096u;
                if (lane == 0) bulk_wait_read<1>();  // the box that used `buf` two stores ago has been read
                __syncwarp();
                if (g.transpose_out) {
                    // D^T tile: lane = output column (TMEM lane), register p = output row (pixel);
                    // box row p, column lane, 128B-swizzled: conflict-free 4-byte stores
                    uint8_t *bp = smem_raw + (buf - raw) + ((lane & 3) << 2);
#pragma unroll
                    for (int pr = 0; pr < 32; ++pr)
                        *reinterpret_cast<uint32_t *>(bp + pr * 128 + ((((lane >> 2) ^ (pr & 7))) << 4)) = r[pr];
                } else {
                    uint8_t *rowp = smem_raw + (buf - raw) + lane * 128;
#pragma unroll
                    for (int j = 0; j < 8; ++j)
                        *reinterpret_cast<uint4 *>(rowp + ((j ^ (lane & 7)) << 4)) =
                            make_uint4(r[4 * j], r[4 * j + 1], r[4 * j + 2], r[4 * j + 3]);
                }
                fence_async_shared();
                __syncwarp();
                if (lane == 0 && g.transpose_out) {
                    tma_store_3d(&tcm, buf, row0, 0, tc.n_t * BN + c * 32);
                    bulk_commit();
                } else if (lane == 0) {
                    const int col0 = tc.n_t * BN + c * 32;
                    if (g.store_mode == STORE_ATOMIC_ADD)
                        tma_reduce_add_3d(&tcm, buf, col0, tc.tap, row0);
                    else if (g.store_mode == STORE_SLICE_ADD)
                        tma_reduce_add_3d(&tcm, buf, col0, tc.split, row0);
                    else
                        tma_store_3d(&tcm, buf, col0, g.store_mode == STORE_SPLIT ? tc.split : tc.tap, row0);
                    bulk_commit();
                }
                ++nbox;
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(tempty_bar(acc));
            acc ^= 1;
            if (acc == 0) acc_phase ^= 1u;
        }
        if (lane == 0) bulk_wait<0>();
    }
    if (g.stats && lane == 0) {
        // slots: 0 producer<-empty, 1 MMA<-tempty, 2 epilogue<-tfull (sum of 4 warps), 3 CTA cycles,
        // 4 MMA<-full (TMA data)
        const int slot = warp == 0 ? 0 : (warp == 1 ? 1 : 2);
        atomicAdd(g.stats + slot, w_stat);
        if (warp == 0) atomicAdd(g.stats + 3, (unsigned long long)(clock64() - t_start));
    }
    tc_fence_before();
    __syncthreads();
    if (CS > 1) cluster_sync_all();  // no CTA leaves while peers may still signal its barriers
    tc_fence_after();
    if (warp == 1) tmem_dealloc<Cfg::TMEM_COLS>(tmem_base);
}

// ------------------------------------------------------------------------------------ host side
typedef CUresult (*PFN_encodeTiled_t)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                      const cuuint64_t *, const cuuint32_t *, const cuuint32_t *,
                                      CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion,
                                      CUtensorMapFloatOOBfill);

static PFN_encodeTiled_t encode_fn() {
    static PFN_encodeTiled_t fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        cudaDriverEntryPointQueryResult q;
        void *p = nullptr;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_encodeTiled_t>(p);
    });
    return fn;
}

bool make_map_2d(CUtensorMap *m, const void *ptr, uint64_t inner, uint64_t outer, uint32_t box_inner,
                 uint32_t box_outer) {
    auto fn = encode_fn();
    if (!fn) return false;
    if ((inner * 2) % 16 != 0 || (reinterpret_cast<uintptr_t>(ptr) & 15)) return false;
    cuuint64_t dims[2] = {inner, outer};
    cuuint64_t strides[1] = {inner * 2};
    cuuint32_t box[2] = {box_inner, box_outer};
    cuuint32_t es[2] = {1, 1};
    return fn(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void *>(ptr), dims, strides, box, es,
              CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// fp32 output viewed as [rows][taps][cols] (row pitch ldc, tap pitch tap_pitch floats), box 32 x 1 x 32.
static bool make_map_out(CUtensorMap *m, float *ptr, uint64_t cols, uint64_t taps, uint64_t rows, uint64_t tap_pitch,
                         uint64_t ldc) {
    auto fn = encode_fn();
    if (!fn) return false;
    if ((ldc * 4) % 16 || (tap_pitch * 4) % 16 || (reinterpret_cast<uintptr_t>(ptr) & 15)) return false;
    cuuint64_t dims[3] = {cols, taps, rows};
    cuuint64_t strides[2] = {tap_pitch * 4, ldc * 4};
    cuuint32_t box[3] = {32, 1, 32};
    cuuint32_t es[3] = {1, 1, 1};
    return fn(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, ptr, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
              CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

bool make_map_conv(CUtensorMap *m, const void *ptr, uint64_t C, uint64_t W, uint64_t H, uint64_t NB,
                   uint32_t box_w, uint32_t box_h, uint32_t box_n) {
    auto fn = encode_fn();
    if (!fn) return false;
    if ((C * 2) % 16 != 0 || (reinterpret_cast<uintptr_t>(ptr) & 15)) return false;
    cuuint64_t dims[4] = {C, W, H, NB};
    cuuint64_t strides[3] = {C * 2, W * C * 2, H * W * C * 2};
    cuuint32_t box[4] = {64, box_w, box_h, box_n};
    cuuint32_t es[4] = {1, 1, 1, 1};
    return fn(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, const_cast<void *>(ptr), dims, strides, box, es,
              CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// 4D NHWC map with a box of `cin_box` channels (32/64/128 bytes -> matching swizzle) and element strides
static bool make_map_conv_s(CUtensorMap *m, const void *ptr, uint64_t C, uint64_t W, uint64_t H, uint64_t NB,
                            uint32_t cin_box, uint32_t box_w, uint32_t box_h, uint32_t box_n, uint32_t stride) {
    auto fn = encode_fn();
    if (!fn) return false;
    if ((C * 2) % 16 != 0 || (reinterpret_cast<uintptr_t>(ptr) & 15)) return false;
    cuuint64_t dims[4] = {C, W, H, NB};
    cuuint64_t strides[3] = {C * 2, W * C * 2, H * W * C * 2};
    cuuint32_t box[4] = {cin_box, box_w * stride, box_h * stride, box_n};
    cuuint32_t es[4] = {1, stride, stride, 1};
    const CUtensorMapSwizzle sw = cin_box == 16 ? CU_TENSOR_MAP_SWIZZLE_32B
                                  : cin_box == 32 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_128B;
    return fn(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, const_cast<void *>(ptr), dims, strides, box, es,
              CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// 2D K-major map [outer][inner] with a box of `box_inner` elements and the matching swizzle
static bool make_map_2d_sw(CUtensorMap *m, const void *ptr, uint64_t inner, uint64_t outer, uint32_t box_inner,
                           uint32_t box_outer) {
    auto fn = encode_fn();
    if (!fn) return false;
    if ((inner * 2) % 16 != 0 || (reinterpret_cast<uintptr_t>(ptr) & 15)) return false;
    cuuint64_t dims[2] = {inner, outer};
    cuuint64_t strides[1] = {inner * 2};
    cuuint32_t box[2] = {box_inner, box_outer};
    cuuint32_t es[2] = {1, 1};
    const CUtensorMapSwizzle sw = box_inner == 16 ? CU_TENSOR_MAP_SWIZZLE_32B
                                  : box_inner == 32 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_128B;
    return fn(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void *>(ptr), dims, strides, box, es,
              CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

static int pick_bn(int N) { return N <= 64 ? 64 : (N <= 128 ? 128 : 256); }

// Cluster size for B multicast (K-major, unsplit GEMMs with enough M tiles).  SKIPPER_GEMM_CS
// overrides the default (1, 2 or 4).
static int pick_cs(const GemmDev &d) {
    static int def = -1;
    if (def < 0) {
        const char *e = getenv("SKIPPER_GEMM_CS");
        def = e ? atoi(e) : 2;
        if (def != 1 && def != 2 && def != 4) def = 2;
    }
    if (d.splits != 1 || d.taps != 1 || d.m_tiles < 2 * def) return 1;
    return def;
}
static int cdiv(long long a, long long b) { return (int)((a + b - 1) / b); }

// box geometry covering `rows` consecutive flat rows of an [nb][h][w] image stack
static bool conv_box(int h, int w, int rows, uint32_t *bw, uint32_t *bh, uint32_t *bn) {
    if (w > rows || rows % w) return false;
    int by = rows / w;
    if (by <= h) {
        if (h % by) return false;
        *bw = w; *bh = by; *bn = 1;
        return true;
    }
    if (by % h) return false;
    *bw = w; *bh = h; *bn = by / h;
    return *bn <= 256;
}

bool plan_fc(GemmLaunch *g, const void *A, const void *B, float *C, int M, int N, int K, int splits) {
    if (M <= 0 || N <= 0 || K <= 0 || N % 4 || K % 8) return false;
    GemmDev &d = g->d;
    d = GemmDev{};
    g->bn = pick_bn(N);
    g->mn_major = 0;
    d.m_tiles = cdiv(M, BM);
    d.n_tiles = cdiv(N, g->bn);
    d.taps = 1;
    d.splits = 1;
    d.num_kb = cdiv(K, BK);
    if (splits < 1) splits = 1;
    if (splits > d.num_kb) splits = d.num_kb;
    d.kb_per_split = cdiv(d.num_kb, splits);
    d.splits = cdiv(d.num_kb, d.kb_per_split);
    d.a_kind = OP_K2D;
    d.b_kind = OP_K2D;
    d.C = C;
    d.ldc = N;
    d.M = M;
    d.N = N;
    d.store_mode = d.splits > 1 ? STORE_SPLIT : STORE_OVERWRITE;
    d.cols_per_tap = 0;
    g->cs = pick_cs(d);
    // output viewed as [M][splits][N]: slice s at C + s*M*N
    return make_map_2d(&g->ta, A, K, M, BK, BM) && make_map_2d(&g->tb, B, K, N, BK, g->bn / g->cs) &&
           make_map_out(&g->tc, C, N, d.splits, M, (uint64_t)M * N, N);
}

// fit = true: at most mult * num_sms units (floor), so a one-unit-per-CTA launch has no second wave
static void choose_splits(GemmDev &d, int base_tiles, int num_sms, int mult = 2, bool fit = false) {
    if (getenv("SKIPPER_SPLIT_MULT")) mult = atoi(getenv("SKIPPER_SPLIT_MULT"));  // experiments
    int target = mult * num_sms;
    int splits = base_tiles >= target ? 1 : (fit ? target / base_tiles : cdiv(target, base_tiles));
    if (splits > d.num_kb) splits = d.num_kb;
    if (splits < 1) splits = 1;
    d.kb_per_split = cdiv(d.num_kb, splits);
    d.splits = cdiv(d.num_kb, d.kb_per_split);
}

// split-K units per SM of the deterministic (slice) weight gradients: every split adds its whole output
// tile into its own slice, so the slice bytes grow with the split count (SKIPPER_WG_SLICE_MULT, experiments)
static int slice_mult(int dflt) {
    static int m = -1;
    if (m < 0) {
        const char *e = getenv("SKIPPER_WG_SLICE_MULT");
        m = e ? std::max(1, atoi(e)) : 0;
    }
    return m ? m : dflt;
}

// The bound on the split count before choose_splits rounds it to whole K blocks per split (the rounded
// count is not monotone in M; this bound is, and every launch at a smaller M splits at most this often)
static int splits_bound(long long M, int base_tiles, int num_sms, int mult) {
    if (getenv("SKIPPER_SPLIT_MULT")) mult = atoi(getenv("SKIPPER_SPLIT_MULT"));
    const int target = mult * num_sms;
    int s = base_tiles >= target ? 1 : target / base_tiles;
    return std::max(1, (int)std::min<long long>(s, cdiv(M, BK)));
}

int fc_wgrad_splits(long long M, int N, int K, int num_sms) {
    return splits_bound(M, cdiv(N, BM) * cdiv(K, pick_bn(K)), num_sms, slice_mult(1));
}

static int conv_wgrad_bn(int cin) {
    int bn = (9 * cin) % 256 && (9 * cin) % 192 == 0 ? 192 : 256;
    if (getenv("SKIPPER_WG_BN")) bn = atoi(getenv("SKIPPER_WG_BN"));  // experiments
    return bn;
}

int conv_wgrad_splits(long long M, int cin, int cout, int num_sms) {
    return splits_bound(M, cdiv(cout, BM) * cdiv(9LL * cin, conv_wgrad_bn(cin)), num_sms, slice_mult(1));
}

bool plan_fc_wgrad(GemmLaunch *g, const void *D, const void *X, float *dW, int M, int N, int K, int num_sms,
                   int slices) {
    // GEMM rows = N (output neurons), GEMM cols = K (inputs), reduction over M rows.
    if (M <= 0 || N <= 0 || K <= 0 || N % 8 || K % 8) return false;
    GemmDev &d = g->d;
    d = GemmDev{};
    g->bn = pick_bn(K);
    g->mn_major = 1;
    g->cs = 1;
    d.m_tiles = cdiv(N, BM);
    d.n_tiles = cdiv(K, g->bn);
    d.taps = 1;
    d.num_kb = cdiv(M, BK);
    choose_splits(d, d.m_tiles * d.n_tiles, num_sms, slices > 0 ? slice_mult(1) : 2, slices > 0);
    if (slices > 0 && d.splits > slices) return false;
    d.a_kind = OP_MN2D;
    d.b_kind = OP_MN2D;
    d.C = dW;
    d.ldc = K;
    d.M = N;
    d.N = K;
    d.store_mode = slices > 0 ? STORE_SLICE_ADD : STORE_ATOMIC_ADD;
    return make_map_2d(&g->ta, D, N, M, 64, BK) && make_map_2d(&g->tb, X, K, M, 64, BK) &&
           make_map_out(&g->tc, dW, K, slices > 0 ? slices : 1, N, (uint64_t)N * K, K);
}

bool plan_conv(GemmLaunch *g, const void *X, const void *Wk, float *Y, int nb, int h, int w, int cin, int cout,
               int sign) {
    // forward: A = X (cin channels), B = Wk [cout][9*cin], out channels cout.
    // dgrad (sign = -1): caller passes X = D (cout channels of the layer) as "cin" and Wt as Wk.
    if (cin % 64 || cout % 8) return false;
    uint32_t tw, th, tn;
    if (cout <= 128 && conv_box(h, w, 256, &tw, &th, &tn)) {
        // Narrow output: compute Y^T = Wk . X^T so the pixels are the 256-wide N side of the tile
        // (128 x 256 tiles run the tensor cores far better than 128 x 128 / 128 x 64 ones).
        const long long M = (long long)nb * h * w;
        GemmDev &d = g->d;
        d = GemmDev{};
        g->bn = 256;
        g->mn_major = 0;
        g->cs = 1;
        d.m_tiles = 1;
        d.n_tiles = cdiv(M, 256);
        d.taps = 1;
        d.splits = 1;
        d.conv_cb = cin / 64;
        d.num_kb = 9 * d.conv_cb;
        d.kb_per_split = d.num_kb;
        d.a_kind = OP_K2D;
        d.b_kind = OP_KCONV;
        d.conv_hw = h * w;
        d.conv_w = w;
        d.conv_sign = sign;
        d.transpose_out = 1;
        d.C = Y;
        d.ldc = cout;
        d.M = cout;
        d.N = (int)M;
        d.store_mode = STORE_OVERWRITE;
        return make_map_2d(&g->ta, Wk, 9ull * cin, cout, BK, BM) && make_map_conv(&g->tb, X, cin, w, h, nb, tw, th, tn) &&
               make_map_out(&g->tc, Y, cout, 1, M, cout, cout);
    }
    uint32_t bw, bh, bnn;
    if (!conv_box(h, w, BM, &bw, &bh, &bnn)) return false;
    const long long M = (long long)nb * h * w;
    GemmDev &d = g->d;
    d = GemmDev{};
    g->bn = pick_bn(cout);
    g->mn_major = 0;
    d.m_tiles = cdiv(M, BM);
    d.n_tiles = cdiv(cout, g->bn);
    d.taps = 1;
    d.splits = 1;
    d.conv_cb = cin / 64;
    d.num_kb = 9 * d.conv_cb;
    d.kb_per_split = d.num_kb;
    d.a_kind = OP_KCONV;
    d.b_kind = OP_K2D;
    d.conv_hw = h * w;
    d.conv_w = w;
    d.conv_sign = sign;
    d.C = Y;
    d.ldc = cout;
    d.M = (int)M;
    d.N = cout;
    d.store_mode = STORE_OVERWRITE;
    g->cs = pick_cs(d);
    return make_map_conv(&g->ta, X, cin, w, h, nb, bw, bh, bnn) && make_map_2d(&g->tb, Wk, 9ull * cin, cout, BK, g->bn / g->cs) &&
           make_map_out(&g->tc, Y, cout, 1, M, cout, cout);
}

bool plan_conv_s(GemmLaunch *g, const void *X, const void *Wk, float *Y, int nb, int h, int w, int cin, int cout,
                 int sign, int stride) {
    if (cout % 8 || (stride != 1 && stride != 2) || (sign == -1 && stride != 1)) return false;
    int kblk, cb;
    if (cin == 16 || cin == 32) {
        kblk = cin;
        cb = 1;
    } else if (cin % 64 == 0) {
        kblk = 64;
        cb = cin / 64;
    } else {
        return false;
    }
    uint32_t bw, bh, bnn;
    if (!conv_box(h, w, BM, &bw, &bh, &bnn)) return false;
    if (bw * stride > 256 || bh * stride > 256) return false;
    const long long M = (long long)nb * h * w;
    GemmDev &d = g->d;
    d = GemmDev{};
    g->bn = pick_bn(cout);
    g->mn_major = 0;
    g->cs = 1;
    d.m_tiles = cdiv(M, BM);
    d.n_tiles = cdiv(cout, g->bn);
    d.taps = 1;
    d.splits = 1;
    d.conv_cb = cb;
    d.num_kb = 9 * cb;
    d.kb_per_split = d.num_kb;
    d.a_kind = OP_KCONV;
    d.b_kind = OP_K2D;
    d.conv_hw = h * w;
    d.conv_w = w;
    d.conv_sign = sign;
    d.conv_stride = stride;
    d.kblk = kblk;
    d.stage_tx = (uint32_t)(BM + g->bn) * kblk * 2;
    d.stage_stride = (d.stage_tx + 1023u) & ~1023u;
    d.ring = (int)std::min<uint32_t>(GemmCfg<64>::MAX_RING, (uint32_t)(192u * 1024u) / d.stage_stride);
    d.C = Y;
    d.ldc = cout;
    d.M = (int)M;
    d.N = cout;
    d.store_mode = STORE_OVERWRITE;
    return make_map_conv_s(&g->ta, X, cin, (uint64_t)w * stride, (uint64_t)h * stride, nb, kblk, bw, bh, bnn, stride) &&
           make_map_2d_sw(&g->tb, Wk, 9ull * cin, cout, kblk, g->bn) && make_map_out(&g->tc, Y, cout, 1, M, cout, cout);
}

bool plan_conv_wgrad(GemmLaunch *g, const void *D, const void *X, float *dW, int nb, int h, int w, int cin, int cout,
                     int num_sms, int slices) {
    if (cin % 64 || cout % 8) return false;
    uint32_t bw, bh, bnn;
    if (!conv_box(h, w, BK, &bw, &bh, &bnn)) return false;
    const long long M = (long long)nb * h * w;
    GemmDev &d = g->d;
    d = GemmDev{};
    // N = (tap, cin) = 9*cin columns in 256-wide tiles (192-wide when that tiles 9*cin exactly and 256
    // does not: cin = 64 -> 3 x 192 instead of 3 x 256 with a quarter-full last tile); each 64-column
    // chunk is one tap's shifted box
    g->bn = conv_wgrad_bn(cin);
    g->mn_major = 1;
    g->cs = 1;
    d.m_tiles = cdiv(cout, BM);
    d.n_tiles = cdiv(9LL * cin, g->bn);
    d.taps = 1;
    d.wg_cin = cin;
    d.num_kb = cdiv(M, BK);
    // ~4 units per CTA with reduce-add into one dW: measured +5-15 % over 2; slices: slice_mult
    choose_splits(d, d.m_tiles * d.n_tiles, num_sms, slices > 0 ? slice_mult(1) : 4, slices > 0);
    if (slices > 0 && d.splits > slices) return false;
    d.a_kind = OP_MN2D;
    static const bool box4d = getenv("SKIPPER_WG_4D") && atoi(getenv("SKIPPER_WG_4D"));  // experiments
    d.b_kind = box4d ? OP_MNCONV : OP_MNSHIFT;
    d.conv_hw = h * w;
    d.conv_w = w;
    d.conv_sign = 1;
    d.cols_per_tap = 0;
    d.C = dW;
    d.ldc = 9ll * cin;
    d.M = cout;
    d.N = 9 * cin;
    d.store_mode = slices > 0 ? STORE_SLICE_ADD : STORE_ATOMIC_ADD;
    const bool okb = box4d ? make_map_conv(&g->tb, X, cin, w, h, nb, bw, bh, bnn)
                           : make_map_2d(&g->tb, X, cin, (uint64_t)M, 64, BK);
    return make_map_2d(&g->ta, D, cout, M, 64, BK) && okb &&
           make_map_out(&g->tc, dW, 9ull * cin, slices > 0 ? slices : 1, cout, 9ull * cin * cout, 9ull * cin);
}

template <int BN, int MN, int CS>
static cudaError_t launch_t(const GemmLaunch &g, cudaStream_t stream, int num_sms) {
    using Cfg = GemmCfg<BN>;
    auto kern = gemm_tc_kernel<BN, MN, CS>;
    static int max_clusters = -1;
    if (max_clusters < 0) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)Cfg::SMEM_BYTES);
        if (e != cudaSuccess) return e;
        max_clusters = num_sms / CS;
        if (CS > 1) {
            cudaLaunchConfig_t qc{};
            qc.gridDim = dim3(CS * max_clusters);
            qc.blockDim = dim3(kThreads<MN>);
            qc.dynamicSmemBytes = Cfg::SMEM_BYTES;
            cudaLaunchAttribute at[1];
            at[0].id = cudaLaunchAttributeClusterDimension;
            at[0].val.clusterDim.x = CS;
            at[0].val.clusterDim.y = 1;
            at[0].val.clusterDim.z = 1;
            qc.attrs = at;
            qc.numAttrs = 1;
            int n = 0;
            if (cudaOccupancyMaxActiveClusters(&n, kern, &qc) == cudaSuccess && n > 0) max_clusters = n;
            cudaGetLastError();
        }
    }
    const int total = CS > 1 ? ((g.d.m_tiles + CS - 1) / CS) * g.d.n_tiles : g.d.m_tiles * g.d.n_tiles * g.d.taps * g.d.splits;
    const int units = total < max_clusters ? total : max_clusters;
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(units * CS);
    cfg.blockDim = dim3(kThreads<MN>);
    cfg.dynamicSmemBytes = Cfg::SMEM_BYTES;
    cfg.stream = stream;
    cudaLaunchAttribute attrs[2];
    attrs[0].id = cudaLaunchAttributeClusterDimension;
    attrs[0].val.clusterDim.x = CS;
    attrs[0].val.clusterDim.y = 1;
    attrs[0].val.clusterDim.z = 1;
    attrs[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attrs[1].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
    cfg.attrs = attrs;
    cfg.numAttrs = 2;
    return cudaLaunchKernelEx(&cfg, kern, g.ta, g.tb, g.tc, g.d);
}

cudaError_t gemm_run(const GemmLaunch &g, cudaStream_t stream, int num_sms) {
    const int total = g.d.m_tiles * g.d.n_tiles * g.d.taps * g.d.splits;
    if (total <= 0) return cudaSuccess;
    if (g.mn_major) {
        if (g.bn == 64) return launch_t<64, 1, 1>(g, stream, num_sms);
        if (g.bn == 128) return launch_t<128, 1, 1>(g, stream, num_sms);
        if (g.bn == 192) return launch_t<192, 1, 1>(g, stream, num_sms);
        return launch_t<256, 1, 1>(g, stream, num_sms);
    }
    if (g.cs == 4) {
        if (g.bn == 64) return launch_t<64, 0, 4>(g, stream, num_sms);
        if (g.bn == 128) return launch_t<128, 0, 4>(g, stream, num_sms);
        return launch_t<256, 0, 4>(g, stream, num_sms);
    }
    if (g.cs == 2) {
        if (g.bn == 64) return launch_t<64, 0, 2>(g, stream, num_sms);
        if (g.bn == 128) return launch_t<128, 0, 2>(g, stream, num_sms);
        return launch_t<256, 0, 2>(g, stream, num_sms);
    }
    if (g.bn == 64) return launch_t<64, 0, 1>(g, stream, num_sms);
    if (g.bn == 128) return launch_t<128, 0, 1>(g, stream, num_sms);
    return launch_t<256, 0, 1>(g, stream, num_sms);
}

bool pdl_enabled() {
    static const bool on = !(getenv("SKIPPER_NO_PDL") && atoi(getenv("SKIPPER_NO_PDL")));
    return on;
}

int device_num_sms() {
    static int n = 0;
    if (n == 0) {
        int dev = 0;
        cudaGetDevice(&dev);
        if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || n <= 0) n = 148;
    }
    return n;
}

}  // namespace sk
