// layer0.cu - fused first spiking layer for narrow inputs (RGB frames, DVS polarity channels).
//
// One kernel does, for a segment's rows (timesteps) of a 3x3 / pad-1 conv layer with 9*C0 <= 32:
//   im2col of the uint8 input spikes built directly in shared memory (producer warps),
//   the synaptic current I = W o^0 on the tensor cores (tcgen05.mma M=128, N=Cout, K=32, bf16 in,
//   fp32 accumulate in TMEM, double-buffered accumulators),
//   the LIF recurrence of Eq.1 in the epilogue with the membrane state held in
//   registers across the rows (one thread = one pixel x all Cout channels),
//   2x2 average pooling of the output spikes through warp shuffles (the 128 tile rows are ordered
//   so that each 2x2 window sits in 4 consecutive lanes), SAM spike counts (Eq.4) for
//   the input and this layer, checkpoint write at the segment start, stored U (recompute/full).
// The currents never touch HBM: per neuron-step only the layer output (0.5 B pooled) and, when
// stored, U (4 B) are written.
#include "common.cuh"
#include "kernels.h"

namespace sk {

// warps 0-3: producers (one tile row each), warp 4: MMA issuer + TMEM owner,
// warps 5..: epilogue, 4 per 32-channel chunk (warp w reads TMEM lane quadrant w % 4)
static constexpr int L0_PROD_WARPS = 4;
static constexpr int L0_MMA_WARP = 4;
static constexpr int L0_EPI_WARP0 = 5;
static constexpr int L0_STAGES = 4;
static constexpr uint32_t L0_A_BYTES = 128 * 32 * 2;  // 128 rows x K=32 bf16
static constexpr uint32_t L0_PLANE_A = 128 * 16;      // one 8-column K chunk of all 128 rows

SK_DEV float lif_step0(float U, float I, float o, float lam, float th) {
    return __fsub_rn(__fadd_rn(__fmul_rn(lam, U), I), __fmul_rn(th, o));
}

// UMMA descriptor, no swizzle, K-major: 16-byte rows (8 bf16 of K) contiguous within an 8-row core
// matrix, core matrices SBO = 128 B apart along M/N, K chunks LBO bytes apart.
SK_DEV uint64_t umma_desc_noswz(uint32_t saddr, uint32_t lbo_bytes) {
    uint64_t d = 0;
    d |= (uint64_t)((saddr >> 4) & 0x3FFF);
    d |= (uint64_t)((lbo_bytes >> 4) & 0x3FFF) << 16;
    d |= (uint64_t)(128u >> 4) << 32;
    d |= (uint64_t)1 << 46;
    return d;  // layout type 0 = SWIZZLE_NONE
}

struct L0Tile {
    int tiles_b, tiles_y, tiles_x;  // tile grid
    int TB, TH, TW;                 // tile extent (images, rows, cols): TB*TH*TW = 128
};

// tile row r -> (image offset, y offset, x offset) within the tile
SK_DEV void l0_row_pos(const L0Tile &g, int pool, int r, int &bl, int &yl, int &xl) {
    if (pool) {
        const int q = r >> 2, sub = r & 3;
        const int QW = g.TW >> 1, QH = g.TH >> 1;
        const int qx = q % QW, qy = (q / QW) % QH;
        bl = q / (QW * QH);
        yl = 2 * qy + (sub >> 1);
        xl = 2 * qx + (sub & 1);
    } else {
        xl = r % g.TW;
        yl = (r / g.TW) % g.TH;
        bl = r / (g.TW * g.TH);
    }
}

template <int NCH>  // Cout = 32 * NCH
__global__ void __launch_bounds__(32 * (L0_EPI_WARP0 + 4 * NCH), 1) layer0_fwd_kernel(const L0FwdArgs a, const L0Tile tg) {
    constexpr int N = 32 * NCH;
    constexpr uint32_t PLANE_B = N * 16;
    constexpr uint32_t TMEM_COLS = (2 * N <= 64) ? 64 : (2 * N <= 128 ? 128 : 256);
    extern __shared__ uint8_t smem_raw[];
    const uint32_t raw = smem_u32(smem_raw);
    const uint32_t base = (raw + 1023u) & ~1023u;
    const uint32_t sA = base;                                 // L0_STAGES x 8 KB
    const uint32_t sB = sA + L0_STAGES * L0_A_BYTES;          // N x 32 bf16
    const uint32_t bars = sB + 4 * PLANE_B;
    auto full_bar = [&](int s) { return bars + 8u * s; };
    auto empty_bar = [&](int s) { return bars + 8u * (L0_STAGES + s); };
    auto tfull_bar = [&](int i) { return bars + 8u * (2 * L0_STAGES + i); };
    auto tempty_bar = [&](int i) { return bars + 8u * (2 * L0_STAGES + 2 + i); };
    const uint32_t tmem_slot = bars + 8u * (2 * L0_STAGES + 4);
    unsigned *row_cnt = reinterpret_cast<unsigned *>(smem_raw + (tmem_slot + 16 - raw));
    uint8_t *sB_ptr = smem_raw + (sB - raw);
    uint8_t *sA_ptr = smem_raw + (sA - raw);

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int HW = a.H * a.W;
    const int tiles = tg.tiles_b * tg.tiles_y * tg.tiles_x;
    const int r_mma0 = a.restore ? 1 : 0;

    // weights -> smem (no-swizzle K-major core matrices), row counters
    for (int i = threadIdx.x; i < N * 32; i += blockDim.x) {
        const int n = i >> 5, k = i & 31;
        *reinterpret_cast<uint16_t *>(sB_ptr + (k >> 3) * PLANE_B + n * 16 + (k & 7) * 2) = a.wbp[n * 32 + k];
    }
    for (int r = threadIdx.x; r < a.R; r += blockDim.x) row_cnt[r] = 0;
    fence_async_shared();
    if (threadIdx.x == 0) {
        for (int s = 0; s < L0_STAGES; ++s) {
            mbar_init(full_bar(s), L0_PROD_WARPS);
            mbar_init(empty_bar(s), 1);
        }
        for (int i = 0; i < 2; ++i) {
            mbar_init(tfull_bar(i), 1);
            mbar_init(tempty_bar(i), 4 * NCH);
        }
        fence_mbar_init();
    }
    if (warp == L0_MMA_WARP) tmem_alloc<TMEM_COLS>(tmem_slot);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *reinterpret_cast<volatile uint32_t *>(smem_raw + (tmem_slot - raw));

    auto tile_origin = [&](int tile, int &b0, int &y0, int &x0) {
        const int tx = tile % tg.tiles_x;
        const int ty = (tile / tg.tiles_x) % tg.tiles_y;
        const int tb = tile / (tg.tiles_x * tg.tiles_y);
        b0 = tb * tg.TB;
        y0 = ty * tg.TH;
        x0 = tx * tg.TW;
    };
    auto row_time = [&](int r) -> long long { return a.row_t ? a.row_t[r] : (long long)a.t0 + r; };

    if (warp < L0_PROD_WARPS) {
        // ------------------------------------------------------------ producers: im2col -> smem
        // thread r builds tile row r from three 16-byte windows of the uint8 input rows y-1, y, y+1
        // (loads issued one row ahead of the build so their latency overlaps the barrier waits)
        const int r = threadIdx.x;  // 0..127
        const int rowbytes = a.W * a.C0;
        const int rowwords = rowbytes >> 2;
        int stage = 0;
        uint32_t phase = 0;
        const int nit_tile = a.R - r_mma0;
        auto fetch = [&](int tile, int ri, uint32_t (&wv)[3][4], int &shift, bool &ok, bool &ctr) {
            int b0, y0, x0, bl, yl, xl;
            tile_origin(tile, b0, y0, x0);
            l0_row_pos(tg, a.pool, r, bl, yl, xl);
            const int b = b0 + bl, yy = y0 + yl, xx = x0 + xl;
            ok = b < a.B;
            ctr = ok;
            const long long t = row_time(ri);
            const int bstart = a.C0 * (xx - 1);
            const int w0 = bstart >= 0 ? (bstart >> 2) : -1;
            shift = bstart - 4 * w0;
#pragma unroll
            for (int dy = 0; dy < 3; ++dy) {
                const int y = yy + dy - 1;
                const bool rok = ok && y >= 0 && y < a.H;
                const uint32_t *rowp =
                    reinterpret_cast<const uint32_t *>(a.x + ((t * a.B + (rok ? b : 0)) * a.H + (rok ? y : 0)) * (long long)rowbytes);
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const int wi = w0 + j;
                    wv[dy][j] = (rok && wi >= 0 && wi < rowwords) ? __ldg(rowp + wi) : 0u;
                }
            }
        };
        uint32_t nx[3][4];
        int nshift = 0;
        bool nok = false, nctr = false;
        int tile = blockIdx.x, ri = r_mma0;
        if (tile < tiles && nit_tile > 0) fetch(tile, ri, nx, nshift, nok, nctr);
        while (tile < tiles && nit_tile > 0) {
            uint32_t cw[3][4];
#pragma unroll
            for (int dy = 0; dy < 3; ++dy)
#pragma unroll
                for (int j = 0; j < 4; ++j) cw[dy][j] = nx[dy][j];
            const int cshift = nshift;
            const bool cok = nok;
            const int cri = ri;
            // advance and prefetch the next row
            if (++ri == a.R) {
                ri = r_mma0;
                tile += gridDim.x;
            }
            if (tile < tiles) fetch(tile, ri, nx, nshift, nok, nctr);
            // build the im2col row: bit (dy*3+dx)*C0+ci <- window byte dx*C0+ci of row dy
            uint32_t m = 0;
            unsigned cnt = 0;
            if (cok) {
#pragma unroll
                for (int dy = 0; dy < 3; ++dy) {
                    const uint32_t v0 = __funnelshift_r(cw[dy][0], cw[dy][1], 8 * cshift);
                    const uint32_t v1 = __funnelshift_r(cw[dy][1], cw[dy][2], 8 * cshift);
                    const uint32_t v2 = __funnelshift_r(cw[dy][2], cw[dy][3], 8 * cshift);
                    const uint32_t v[3] = {v0, v1, v2};
#pragma unroll
                    for (int j = 0; j < 9; ++j) {  // 3*C0 <= 9 window bytes of this input row
                        if (j < 3 * a.C0) {
                            const uint32_t nz = ((v[j >> 2] >> (8 * (j & 3))) & 0xFFu) ? 1u : 0u;
                            m |= nz << (dy * 3 * a.C0 + j);
                            if (dy == 1) cnt += (j >= a.C0 && j < 2 * a.C0) ? nz : 0u;
                        }
                    }
                }
            }
            mbar_wait(empty_bar(stage), phase ^ 1u);
            uint8_t *dst = sA_ptr + stage * L0_A_BYTES + r * 16;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                uint32_t w[4];
#pragma unroll
                for (int e = 0; e < 4; ++e) {
                    const int k = 8 * j + 2 * e;
                    w[e] = (((m >> k) & 1u) ? 0x3F80u : 0u) | (((m >> (k + 1)) & 1u) ? 0x3F800000u : 0u);
                }
                *reinterpret_cast<uint4 *>(dst + j * L0_PLANE_A) = make_uint4(w[0], w[1], w[2], w[3]);
            }
            if (a.s_part) {
                const unsigned v = __reduce_add_sync(0xffffffffu, cnt);
                if (lane == 0 && v) atomicAdd(&row_cnt[cri], v);
            }
            fence_async_shared();
            __syncwarp();
            if (lane == 0) mbar_arrive(full_bar(stage));
            if (++stage == L0_STAGES) {
                stage = 0;
                phase ^= 1u;
            }
        }
    } else if (warp == L0_MMA_WARP) {
        // ------------------------------------------------------------ MMA issuer
        if (lane == 0) {
            constexpr uint32_t idesc = umma_idesc_bf16(128, N, 0, 0);
            int stage = 0;
            uint32_t phase = 0;
            int acc = 0;
            uint32_t acc_phase = 0;
            for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
                for (int ri = r_mma0; ri < a.R; ++ri) {
                    mbar_wait(tempty_bar(acc), acc_phase ^ 1u);
                    mbar_wait(full_bar(stage), phase);
                    tc_fence_after();
                    const uint32_t a0 = sA + stage * L0_A_BYTES;
#pragma unroll
                    for (int k = 0; k < 2; ++k)
                        tc_mma_f16(tmem_base + acc * N, umma_desc_noswz(a0 + 2 * k * L0_PLANE_A, L0_PLANE_A),
                                   umma_desc_noswz(sB + 2 * k * PLANE_B, PLANE_B), idesc, k ? 1u : 0u);
                    tc_commit(empty_bar(stage));
                    tc_commit(tfull_bar(acc));
                    if (++stage == L0_STAGES) {
                        stage = 0;
                        phase ^= 1u;
                    }
                    acc ^= 1;
                    if (acc == 0) acc_phase ^= 1u;
                }
            }
        }
    } else {
        // ------------------------------------------------------------ epilogue: LIF over rows
        // warp (q, h): TMEM lane quadrant q = warp % 4 (32 tile rows = pixels), channel chunk h
        const int q = warp & 3;
        const int h = (warp - L0_EPI_WARP0) >> 2;
        const int row = q * 32 + lane;
        const long long rs = (long long)a.B * HW * N;
        const int PH = a.pool ? a.H / 2 : a.H, PW = a.pool ? a.W / 2 : a.W;
        const long long ors = (long long)a.B * PH * PW * N;
        const int c0 = h * 32;
        int acc = 0;
        uint32_t acc_phase = 0;
        for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
            int b0, y0, x0, bl, yl, xl;
            tile_origin(tile, b0, y0, x0);
            l0_row_pos(tg, a.pool, row, bl, yl, xl);
            const int b = b0 + bl, yy = y0 + yl, xx = x0 + xl;
            const bool valid = b < a.B;
            const long long pix = ((long long)(valid ? b : 0) * a.H + yy) * a.W + xx;
            const long long opix = a.pool ? ((long long)(valid ? b : 0) * PH + (yy >> 1)) * PW + (xx >> 1) : pix;
            const long long nbase = pix * N + c0;
            float U[32];
            uint32_t ob = 0;
            if (valid) {
#pragma unroll
                for (int c = 0; c < 32; c += 4) {
                    const float4 u = *reinterpret_cast<const float4 *>(a.U_state + nbase + c);
                    U[c] = u.x; U[c + 1] = u.y; U[c + 2] = u.z; U[c + 3] = u.w;
                    const uchar4 o4 = *reinterpret_cast<const uchar4 *>(a.o_state + nbase + c);
                    ob |= (o4.x ? 1u : 0u) << c | (o4.y ? 1u : 0u) << (c + 1) | (o4.z ? 1u : 0u) << (c + 2) |
                          (o4.w ? 1u : 0u) << (c + 3);
                }
            } else {
#pragma unroll
                for (int c = 0; c < 32; ++c) U[c] = 0.f;
            }
            auto store_state = [&](float *Ud, uint8_t *od) {
#pragma unroll
                for (int c = 0; c < 32; c += 4) {
                    *reinterpret_cast<float4 *>(Ud + c) = make_float4(U[c], U[c + 1], U[c + 2], U[c + 3]);
                    *reinterpret_cast<uchar4 *>(od + c) =
                        make_uchar4((ob >> c) & 1u, (ob >> (c + 1)) & 1u, (ob >> (c + 2)) & 1u, (ob >> (c + 3)) & 1u);
                }
            };
            auto emit = [&](int ri) {
                const long long t = row_time(ri);
                unsigned cnt = valid ? __popc(ob) : 0u;
                if (a.pool) {  // 2x2 window = lanes 4k..4k+3
                    const int lb = lane & ~3;
                    const uint32_t w0 = __shfl_sync(0xffffffffu, ob, lb), w1 = __shfl_sync(0xffffffffu, ob, lb + 1);
                    const uint32_t w2 = __shfl_sync(0xffffffffu, ob, lb + 2), w3 = __shfl_sync(0xffffffffu, ob, lb + 3);
                    const uint32_t s0 = w0 ^ w1, cc0 = w0 & w1, s1 = w2 ^ w3, cc1 = w2 & w3;
                    const uint32_t ones = s0 ^ s1, k01 = s0 & s1;
                    const uint32_t twos = cc0 ^ cc1 ^ k01, fours = cc0 & cc1;
                    const int sub = lane & 3;
                    uint32_t pk[4];
                    const uint32_t o8 = (ones >> (sub * 8)) & 0xFFu, t8 = (twos >> (sub * 8)) & 0xFFu;
                    const uint32_t f8 = (fours >> (sub * 8)) & 0xFFu;
#pragma unroll
                    for (int e = 0; e < 4; ++e) {
                        uint32_t v2 = 0;
#pragma unroll
                        for (int hh = 0; hh < 2; ++hh) {
                            const int ch = 2 * e + hh;
                            const uint32_t n = ((o8 >> ch) & 1u) + 2u * ((t8 >> ch) & 1u) + 4u * ((f8 >> ch) & 1u);
                            // n/4 is exact in bf16: its bits are the top half of the fp32 bits
                            v2 |= (__float_as_uint(__uint2float_rn(n) * 0.25f) >> 16) << (16 * hh);
                        }
                        pk[e] = v2;
                    }
                    if (valid)
                        *reinterpret_cast<uint4 *>(a.Po_out + (long long)ri * ors + opix * N + c0 + sub * 8) =
                            make_uint4(pk[0], pk[1], pk[2], pk[3]);
                } else if (valid) {
#pragma unroll
                    for (int j = 0; j < 4; ++j) {
                        uint32_t pk[4];
#pragma unroll
                        for (int e = 0; e < 4; ++e) {
                            const int ch = 8 * j + 2 * e;
                            pk[e] = (((ob >> ch) & 1u) ? 0x3F80u : 0u) | (((ob >> (ch + 1)) & 1u) ? 0x3F800000u : 0u);
                        }
                        *reinterpret_cast<uint4 *>(a.Po_out + (long long)ri * ors + opix * N + c0 + 8 * j) =
                            make_uint4(pk[0], pk[1], pk[2], pk[3]);
                    }
                }
                if (valid) {
                    if (a.U_out) {
#pragma unroll
                        for (int c = 0; c < 32; c += 4)
                            *reinterpret_cast<float4 *>(a.U_out + (long long)ri * rs + nbase + c) =
                                make_float4(U[c], U[c + 1], U[c + 2], U[c + 3]);
                    }
                    if (a.dbg_U) store_state(a.dbg_U + t * rs + nbase, a.dbg_o + t * rs + nbase);
                }
                if (a.s_part) {
                    const unsigned v = __reduce_add_sync(0xffffffffu, cnt);
                    if (lane == 0 && v) atomicAdd(&row_cnt[ri], v);
                }
            };

            if (a.restore) emit(0);
            for (int ri = r_mma0; ri < a.R; ++ri) {
                mbar_wait(tfull_bar(acc), acc_phase);
                tc_fence_after();
                uint32_t r[32];
                tmem_ld_32x32b_x32(tmem_base + ((uint32_t)(q * 32) << 16) + acc * N + c0, r);
                tmem_ld_wait();
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(tempty_bar(acc));
                acc ^= 1;
                if (acc == 0) acc_phase ^= 1u;
                uint32_t nb = 0;
#pragma unroll
                for (int c = 0; c < 32; ++c) {
                    const float u = lif_step0(U[c], __uint_as_float(r[c]), (float)((ob >> c) & 1u), a.lam, a.theta);
                    U[c] = u;
                    nb |= (u > a.theta ? 1u : 0u) << c;
                }
                ob = nb;
                emit(ri);
                if (a.ckU && ri == 0 && valid) store_state(a.ckU + nbase, a.cko + nbase);
            }
            if (!a.restore && valid) store_state(a.U_state + nbase, a.o_state + nbase);
        }
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    if (warp == L0_MMA_WARP) tmem_dealloc<TMEM_COLS>(tmem_base);
    if (a.s_part) {
        for (int r = threadIdx.x; r < a.R; r += blockDim.x) {
            const unsigned v = row_cnt[r];
            if (v) atomicAdd(a.s_part + row_time(r) * 32 + (blockIdx.x & 31), v);
        }
    }
}

static bool l0_tiling(int B, int H, int W, int pool, L0Tile *g) {
    const int HW = H * W;
    if (HW >= 128) {
        int tw = W < 64 ? W : 64;
        while (tw > 1 && (128 % tw || W % tw)) tw >>= 1;
        const int th = 128 / tw;
        if (th > H || H % th || (pool && (th % 2 || tw % 2)) || tw * th != 128) return false;
        g->TB = 1;
        g->TH = th;
        g->TW = tw;
    } else {
        if (128 % HW) return false;
        g->TB = 128 / HW;
        g->TH = H;
        g->TW = W;
        if (pool && (H % 2 || W % 2)) return false;
    }
    g->tiles_b = (B + g->TB - 1) / g->TB;
    g->tiles_y = H / g->TH;
    g->tiles_x = W / g->TW;
    return true;
}

bool layer0_supported(int B, int H, int W, int C0, int N, int pool) {
    L0Tile g;
    return 9 * C0 <= 32 && (N == 32 || N == 64) && (W * C0) % 4 == 0 && l0_tiling(B, H, W, pool, &g);
}

cudaError_t launch_layer0_fwd(const L0FwdArgs &a, cudaStream_t s, int num_sms) {
    L0Tile g;
    if (9 * a.C0 > 32 || !l0_tiling(a.B, a.H, a.W, a.pool, &g)) return cudaErrorInvalidValue;
    const int tiles = g.tiles_b * g.tiles_y * g.tiles_x;
    if (tiles == 0 || a.R == 0) return cudaSuccess;
    const uint32_t smem = 1024 + L0_STAGES * L0_A_BYTES + 4 * a.N * 16 + 8 * (2 * L0_STAGES + 4) + 16 + 4 * a.R;
    const int grid = tiles < num_sms ? tiles : num_sms;
    if (a.W * a.C0 % 4) return cudaErrorInvalidValue;
    if (a.N == 64) {
        static bool set = false;
        if (!set) {
            cudaFuncSetAttribute(layer0_fwd_kernel<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
            set = true;
        }
        layer0_fwd_kernel<2><<<grid, 32 * (L0_EPI_WARP0 + 8), smem, s>>>(a, g);
    } else if (a.N == 32) {
        static bool set = false;
        if (!set) {
            cudaFuncSetAttribute(layer0_fwd_kernel<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
            set = true;
        }
        layer0_fwd_kernel<1><<<grid, 32 * (L0_EPI_WARP0 + 4), smem, s>>>(a, g);
    } else {
        return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

}  // namespace sk

namespace sk {

// ============================================================================ fused layer-0 backward
// Eq.2 reverse scan of the first layer fused with its weight gradient:
//   delta_t = sigma'(U_t) * pool2^T(g_t) + lam * delta_{t+1}   (8 warps, 32 channels each, carry in
//   registers across the kept rows of a tile), bf16(delta) written straight into shared memory as the
//   MN-major A operand of  dW[co][k] += sum_pixels delta[px][co] * im2col(x_t)[px][k]  (tcgen05,
//   M = 128 (Cout 64 used), N = 64 (27 used), K = 128 pixels per row), accumulated in TMEM over all
//   rows of all tiles of the CTA; the im2col operand is built from the uint8 input by 4 producer warps.
// Neither delta nor the im2col rows touch HBM.
static constexpr int LB_STAGES = 4;
static constexpr uint32_t LB_OP_BYTES = 128 * 128;  // 128 pixel lines x 128 B

SK_DEV float surr_grad(float U, float th, int kind, float gamma) {
    if (kind == 0) {
        const float v = 1.0f - fabsf(U - th) / th;
        return v > 0.0f ? gamma * v : 0.0f;
    }
    const float d = 1.0f + gamma * fabsf(U - th);
    return 1.0f / (d * d);
}

__global__ void __launch_bounds__(32 * 13, 1) layer0_bwd_kernel(const L0BwdArgs a, const L0Tile tg) {
    constexpr int N = 64;
    extern __shared__ uint8_t smem_raw[];
    const uint32_t raw = smem_u32(smem_raw);
    const uint32_t base = (raw + 1023u) & ~1023u;
    const uint32_t sA = base;                               // delta^T operands
    const uint32_t sB = sA + LB_STAGES * LB_OP_BYTES;       // im2col^T operands
    const uint32_t bars = sB + LB_STAGES * LB_OP_BYTES;
    auto full_bar = [&](int s) { return bars + 8u * s; };
    auto empty_bar = [&](int s) { return bars + 8u * (LB_STAGES + s); };
    const uint32_t done_bar = bars + 8u * (2 * LB_STAGES);
    const uint32_t tmem_slot = done_bar + 8;
    uint8_t *sA_ptr = smem_raw + (sA - raw);
    uint8_t *sB_ptr = smem_raw + (sB - raw);

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int HW = a.H * a.W;
    const int tiles = tg.tiles_b * tg.tiles_y * tg.tiles_x;

    if (threadIdx.x == 0) {
        for (int s = 0; s < LB_STAGES; ++s) {
            mbar_init(full_bar(s), 4 + 8);  // 4 producer warps + 8 delta warps
            mbar_init(empty_bar(s), 1);
        }
        mbar_init(done_bar, 1);
        fence_mbar_init();
    }
    if (warp == L0_MMA_WARP) tmem_alloc<64>(tmem_slot);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *reinterpret_cast<volatile uint32_t *>(smem_raw + (tmem_slot - raw));

    auto tile_origin = [&](int tile, int &b0, int &y0, int &x0) {
        const int tx = tile % tg.tiles_x;
        const int ty = (tile / tg.tiles_x) % tg.tiles_y;
        const int tb = tile / (tg.tiles_x * tg.tiles_y);
        b0 = tb * tg.TB;
        y0 = ty * tg.TH;
        x0 = tx * tg.TW;
    };
    auto row_time = [&](int r) -> long long { return a.row_t ? a.row_t[r] : (long long)r; };
    // 128B-swizzled position of 16-byte chunk j of pixel line r inside a 128-line operand
    auto line_off = [](int r, int j) -> uint32_t {
        return (uint32_t)((r >> 3) * 1024 + (r & 7) * 128 + ((j ^ (r & 7)) << 4));
    };

    if (warp < 4) {
        // ------------------------------------------------------------ producers: im2col^T lines
        const int r = threadIdx.x;
        const int rowbytes = a.W * a.C0, rowwords = rowbytes >> 2;
        int stage = 0;
        uint32_t phase = 0;
        for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
            int b0, y0, x0, bl, yl, xl;
            tile_origin(tile, b0, y0, x0);
            l0_row_pos(tg, a.pool, r, bl, yl, xl);
            const int b = b0 + bl, yy = y0 + yl, xx = x0 + xl;
            const bool ok = b < a.B;
            const int bstart = a.C0 * (xx - 1);
            const int w0 = bstart >= 0 ? (bstart >> 2) : -1;
            const int shift = bstart - 4 * w0;
            for (int ri = a.R - 1; ri >= 0; --ri) {
                const long long t = row_time(ri);
                uint32_t m = 0;
#pragma unroll
                for (int dy = 0; dy < 3; ++dy) {
                    const int y = yy + dy - 1;
                    const bool rok = ok && y >= 0 && y < a.H;
                    const uint32_t *rowp = reinterpret_cast<const uint32_t *>(
                        a.x + ((t * a.B + (rok ? b : 0)) * a.H + (rok ? y : 0)) * (long long)rowbytes);
                    uint32_t wv[4];
#pragma unroll
                    for (int j = 0; j < 4; ++j) {
                        const int wi = w0 + j;
                        wv[j] = (rok && wi >= 0 && wi < rowwords) ? __ldg(rowp + wi) : 0u;
                    }
                    const uint32_t v[3] = {__funnelshift_r(wv[0], wv[1], 8 * shift), __funnelshift_r(wv[1], wv[2], 8 * shift),
                                           __funnelshift_r(wv[2], wv[3], 8 * shift)};
#pragma unroll
                    for (int j = 0; j < 9; ++j)
                        if (j < 3 * a.C0 && ((v[j >> 2] >> (8 * (j & 3))) & 0xFFu)) m |= 1u << (dy * 3 * a.C0 + j);
                }
                mbar_wait(empty_bar(stage), phase ^ 1u);
                uint8_t *dst = sB_ptr + stage * LB_OP_BYTES;
#pragma unroll
                for (int j = 0; j < 8; ++j) {
                    uint32_t w[4] = {0u, 0u, 0u, 0u};
                    if (j < 4) {
#pragma unroll
                        for (int e = 0; e < 4; ++e) {
                            const int k = 8 * j + 2 * e;
                            w[e] = (((m >> k) & 1u) ? 0x3F80u : 0u) | (((m >> (k + 1)) & 1u) ? 0x3F800000u : 0u);
                        }
                    }
                    *reinterpret_cast<uint4 *>(dst + line_off(r, j)) = make_uint4(w[0], w[1], w[2], w[3]);
                }
                fence_async_shared();
                __syncwarp();
                if (lane == 0) mbar_arrive(full_bar(stage));
                if (++stage == LB_STAGES) {
                    stage = 0;
                    phase ^= 1u;
                }
            }
        }
    } else if (warp == L0_MMA_WARP) {
        // ------------------------------------------------------------ MMA: dW^T tile in TMEM
        if (lane == 0) {
            constexpr uint32_t idesc = umma_idesc_bf16(128, N, 1, 1);
            int stage = 0;
            uint32_t phase = 0;
            bool first = true;
            for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
                for (int ri = a.R - 1; ri >= 0; --ri) {
                    mbar_wait(full_bar(stage), phase);
                    tc_fence_after();
                    const uint32_t a0 = sA + stage * LB_OP_BYTES, b0 = sB + stage * LB_OP_BYTES;
#pragma unroll
                    for (int k = 0; k < 8; ++k) {  // 16 pixels per MMA
                        tc_mma_f16(tmem_base, umma_desc_sw128(a0 + k * 2048u, 0u, 1024u),
                                   umma_desc_sw128(b0 + k * 2048u, 8192u, 1024u), idesc, (first && k == 0) ? 0u : 1u);
                    }
                    first = false;
                    tc_commit(empty_bar(stage));
                    if (++stage == LB_STAGES) {
                        stage = 0;
                        phase ^= 1u;
                    }
                }
            }
            tc_commit(done_bar);
        }
    } else {
        // ------------------------------------------------------------ delta warps
        const int q = warp & 3;
        const int h = (warp - L0_EPI_WARP0) >> 2;
        const int r = q * 32 + lane;
        const int c0 = h * 32;
        const int PH = a.pool ? a.H / 2 : a.H, PW = a.pool ? a.W / 2 : a.W;
        const long long rs = (long long)a.B * HW * N, grs = (long long)a.B * PH * PW * N;
        const float gs = a.pool ? 0.25f : 1.0f;
        int stage = 0;
        uint32_t phase = 0;
        for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
            int b0, y0, x0, bl, yl, xl;
            tile_origin(tile, b0, y0, x0);
            l0_row_pos(tg, a.pool, r, bl, yl, xl);
            const int b = b0 + bl, yy = y0 + yl, xx = x0 + xl;
            const bool ok = b < a.B;
            const long long pix = ((long long)(ok ? b : 0) * a.H + yy) * a.W + xx;
            const long long opix = a.pool ? ((long long)(ok ? b : 0) * PH + (yy >> 1)) * PW + (xx >> 1) : pix;
            float d[32];
#pragma unroll
            for (int c = 0; c < 32; c += 4) {
                const float4 v = ok ? *reinterpret_cast<const float4 *>(a.carry + pix * N + c0 + c) : make_float4(0.f, 0.f, 0.f, 0.f);
                d[c] = v.x; d[c + 1] = v.y; d[c + 2] = v.z; d[c + 3] = v.w;
            }
            for (int ri = a.R - 1; ri >= 0; --ri) {
                float4 uv[8], gv[8];
#pragma unroll
                for (int j = 0; j < 8; ++j) {
                    uv[j] = ok ? __ldg(reinterpret_cast<const float4 *>(a.U + ri * rs + pix * N + c0 + 4 * j)) : make_float4(0.f, 0.f, 0.f, 0.f);
                    gv[j] = ok ? __ldg(reinterpret_cast<const float4 *>(a.g + ri * grs + opix * N + c0 + 4 * j)) : make_float4(0.f, 0.f, 0.f, 0.f);
                }
                uint32_t pk[16];
#pragma unroll
                for (int j = 0; j < 8; ++j) {
                    const float u[4] = {uv[j].x, uv[j].y, uv[j].z, uv[j].w};
                    const float gg[4] = {gv[j].x, gv[j].y, gv[j].z, gv[j].w};
#pragma unroll
                    for (int e = 0; e < 4; ++e) {
                        const int c = 4 * j + e;
                        d[c] = surr_grad(u[e], a.theta, a.surr, a.gamma) * (gs * gg[e]) + a.lam * d[c];
                    }
                    pk[2 * j] = (uint32_t)f2bf_bits(d[4 * j]) | ((uint32_t)f2bf_bits(d[4 * j + 1]) << 16);
                    pk[2 * j + 1] = (uint32_t)f2bf_bits(d[4 * j + 2]) | ((uint32_t)f2bf_bits(d[4 * j + 3]) << 16);
                }
                mbar_wait(empty_bar(stage), phase ^ 1u);
                uint8_t *dst = sA_ptr + stage * LB_OP_BYTES;
#pragma unroll
                for (int j = 0; j < 4; ++j)  // this warp's 32 channels = 16-byte chunks h*4 .. h*4+3
                    *reinterpret_cast<uint4 *>(dst + line_off(r, h * 4 + j)) =
                        ok ? make_uint4(pk[4 * j], pk[4 * j + 1], pk[4 * j + 2], pk[4 * j + 3]) : make_uint4(0u, 0u, 0u, 0u);
                fence_async_shared();
                __syncwarp();
                if (lane == 0) mbar_arrive(full_bar(stage));
                if (++stage == LB_STAGES) {
                    stage = 0;
                    phase ^= 1u;
                }
            }
            if (ok) {
#pragma unroll
                for (int c = 0; c < 32; c += 4)
                    *reinterpret_cast<float4 *>(a.carry + pix * N + c0 + c) = make_float4(d[c], d[c + 1], d[c + 2], d[c + 3]);
            }
        }
        // drain dW^T rows 0..63 (Cout) x columns 0..31 (k) into the fp32 weight gradient
        if (q < 2 && h == 0 && tiles > (int)blockIdx.x) {
            mbar_wait(done_bar, 0);
            tc_fence_after();
            uint32_t v[32];
            tmem_ld_32x32b_x32(tmem_base + ((uint32_t)(q * 32) << 16), v);
            tmem_ld_wait();
            float *dst = a.dW + (long long)(q * 32 + lane) * 32;
#pragma unroll
            for (int k = 0; k < 32; k += 4)
                red_add_v4(dst + k, __uint_as_float(v[k]), __uint_as_float(v[k + 1]), __uint_as_float(v[k + 2]),
                           __uint_as_float(v[k + 3]));
        }
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    if (warp == L0_MMA_WARP) tmem_dealloc<64>(tmem_base);
}

bool layer0_bwd_supported(int B, int H, int W, int C0, int N, int pool) {
    L0Tile g;
    return N == 64 && 9 * C0 <= 32 && (W * C0) % 4 == 0 && l0_tiling(B, H, W, pool, &g);
}

cudaError_t launch_layer0_bwd(const L0BwdArgs &a, cudaStream_t s, int num_sms) {
    L0Tile g;
    if (a.N != 64 || 9 * a.C0 > 32 || !l0_tiling(a.B, a.H, a.W, a.pool, &g)) return cudaErrorInvalidValue;
    const int tiles = g.tiles_b * g.tiles_y * g.tiles_x;
    if (tiles == 0 || a.R == 0) return cudaSuccess;
    const uint32_t smem = 1024 + 2 * LB_STAGES * LB_OP_BYTES + 8 * (2 * LB_STAGES + 1) + 16;
    static bool set = false;
    if (!set) {
        cudaFuncSetAttribute(layer0_bwd_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
        set = true;
    }
    const int grid = tiles < num_sms ? tiles : num_sms;
    layer0_bwd_kernel<<<grid, 32 * 13, smem, s>>>(a, g);
    return cudaGetLastError();
}

}  // namespace sk
