// tma_bench.cu - TMA box-load throughput per SM on B200: 2D boxes vs 4D (NHWC) boxes, in bounds vs
// shifted out of bounds (zero fill), as used by the conv operands.  One CTA per SM, one
// thread issues boxes into a 4-stage ring of 16 KB stages and waits on the stage barriers; the data is
// a small L2-resident tensor so the number measures the TMA path, not HBM.
//
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I../paper_conf_micro_singhslsknnd22_b200/csrc \
//        tools/tma_bench.cu -lcuda -o /tmp/tma_bench
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdint>

#define DEV __device__ __forceinline__
DEV uint32_t su32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
DEV void mbar_init(uint32_t b, uint32_t c) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(b), "r"(c)); }
DEV void mbar_expect(uint32_t b, uint32_t n) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(n) : "memory");
}
DEV void mbar_wait(uint32_t b, uint32_t ph) {
    asm volatile(
        "{\n .reg .pred p;\n W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W;\n}\n" ::"r"(b),
        "r"(ph)
        : "memory");
}
DEV void load2d(uint32_t dst, const CUtensorMap *m, uint32_t bar, int c0, int c1) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(dst),
        "l"((uint64_t)m), "r"(bar), "r"(c0), "r"(c1)
        : "memory");
}
DEV void load4d(uint32_t dst, const CUtensorMap *m, uint32_t bar, int c0, int c1, int c2, int c3) {
    asm volatile(
        "cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6}], [%2];" ::"r"(dst),
        "l"((uint64_t)m), "r"(bar), "r"(c0), "r"(c1), "r"(c2), "r"(c3)
        : "memory");
}

// mode 0: 2D boxes {64, rows}; mode 1: 4D boxes {64, bw, bh, bn} in bounds; mode 2: 4D shifted by (-1, -1)
__global__ void __launch_bounds__(32, 1) bench(const __grid_constant__ CUtensorMap m, int mode, int iters, int nimg,
                                               int H, int W, int bh, int bn, uint32_t box_bytes, long long *cycles) {
    extern __shared__ __align__(1024) uint8_t sm[];
    const uint32_t base = (su32(sm) + 1023u) & ~1023u;
    __shared__ uint64_t bars[4];
    if (threadIdx.x != 0) return;
    for (int s = 0; s < 4; ++s) mbar_init(su32(&bars[s]), 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    const long long t0 = clock64();
    uint32_t ph[4] = {0, 0, 0, 0};
    const int tiles_y = H / bh, tiles_n = nimg / bn;
    for (int i = 0; i < iters + 4; ++i) {
        const int s = i & 3;
        if (i >= 4) {  // wait for the load issued 4 iterations ago into this stage
            mbar_wait(su32(&bars[s]), ph[s]);
            ph[s] ^= 1u;
        }
        if (i < iters) {
            const uint32_t bar = su32(&bars[s]);
            mbar_expect(bar, box_bytes);
            const int t = (int)(blockIdx.x * 7 + i) % (tiles_y * tiles_n);
            const int y0 = (t % tiles_y) * bh, n0 = (t / tiles_y) * bn;
            if (mode == 0)
                load2d(base + s * 16384u, &m, bar, 0, (n0 * H + y0) * W);
            else if (mode == 1)
                load4d(base + s * 16384u, &m, bar, 0, 0, y0, n0);
            else
                load4d(base + s * 16384u, &m, bar, 0, -1, y0 - 1, n0);
        }
    }
    cycles[blockIdx.x] = clock64() - t0;
}

typedef CUresult (*EncodeFn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                             const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                             CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
    EncodeFn enc = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void **)&enc, cudaEnableDefault, &q);
    const int C = 64, sms = 148, iters = 2000;
    long long *cyc;
    cudaMalloc(&cyc, sms * sizeof(long long));
    cudaFuncSetAttribute(bench, cudaFuncAttributeMaxDynamicSharedMemorySize, 4 * 16384 + 1024);
    struct Shape { int H, W, bh, bn, rows; };  // one box = bw=W, bh rows, bn images (or rows for 2D)
    const Shape shapes[] = {{16, 16, 8, 1, 128}, {16, 16, 4, 1, 64}, {4, 4, 4, 8, 128}, {8, 8, 8, 2, 128}, {32, 32, 4, 1, 128}};
    for (const Shape &sh : shapes) {
        const int nimg = 64;
        void *x;
        cudaMalloc(&x, (size_t)nimg * sh.H * sh.W * C * 2);
        cudaMemset(x, 0, (size_t)nimg * sh.H * sh.W * C * 2);
        for (int mode = 0; mode < 3; ++mode) {
            CUtensorMap m;
            uint32_t box_bytes;
            if (mode == 0) {
                cuuint64_t dims[2] = {(cuuint64_t)C, (cuuint64_t)nimg * sh.H * sh.W};
                cuuint64_t str[1] = {(cuuint64_t)C * 2};
                cuuint32_t box[2] = {64, (cuuint32_t)(sh.W * sh.bh * sh.bn)};
                cuuint32_t es[2] = {1, 1};
                enc(&m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, x, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                    CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
                box_bytes = 128u * sh.W * sh.bh * sh.bn;
            } else {
                cuuint64_t dims[4] = {(cuuint64_t)C, (cuuint64_t)sh.W, (cuuint64_t)sh.H, (cuuint64_t)nimg};
                cuuint64_t str[3] = {(cuuint64_t)C * 2, (cuuint64_t)sh.W * C * 2, (cuuint64_t)sh.H * sh.W * C * 2};
                cuuint32_t box[4] = {64, (cuuint32_t)sh.W, (cuuint32_t)sh.bh, (cuuint32_t)sh.bn};
                cuuint32_t es[4] = {1, 1, 1, 1};
                enc(&m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, x, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                    CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
                box_bytes = 128u * sh.W * sh.bh * sh.bn;
            }
            for (int rep = 0; rep < 2; ++rep)
                bench<<<sms, 32, 4 * 16384 + 1024>>>(m, mode, iters, nimg, sh.H, sh.W, sh.bh, sh.bn, box_bytes, cyc);
            cudaError_t e = cudaDeviceSynchronize();
            long long h[148];
            cudaMemcpy(h, cyc, sizeof h, cudaMemcpyDeviceToHost);
            double avg = 0;
            for (int i = 0; i < sms; ++i) avg += (double)h[i] / sms;
            printf("%-22s H=W=%-3d box %5u B (%3d rows): %7.1f cycles/box  %6.1f B/cycle/SM  %s\n",
                   mode == 0 ? "2D" : (mode == 1 ? "4D in-bounds" : "4D shifted (-1,-1)"), sh.H, box_bytes,
                   sh.W * sh.bh * sh.bn, avg / iters, box_bytes * iters / avg, e == cudaSuccess ? "" : cudaGetErrorString(e));
        }
        cudaFree(x);
    }
    return 0;
}
