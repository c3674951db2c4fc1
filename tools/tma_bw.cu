// tma_bw.cu -- per-SM TMA ingest micro-benchmark (tools only; not part of the library).
//
//   nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a tools/tma_bw.cu -o /tmp/tma_bw -lcuda
//   /tmp/tma_bw
//
// Each CTA streams its own slice of a bf16 matrix [rows][cols] (row pitch = cols * 2 B) through
// an S-stage shared-memory ring with 2-D TMA boxes {64 cols, box_rows}, walking like the
// weight operand of a GEMM / LSTM tile: for a block of 128 rows, K-blocks of 64 columns left to
// right.  A consumer thread only waits for each stage and frees it.  Reports aggregate GB/s
// for grid sizes, ring depths and box heights, with the matrix larger than L2 (HBM) and small
// enough to stay in L2.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdint>
#include <vector>

#define CK(x)                                                                              \
    do {                                                                                   \
        cudaError_t e = (x);                                                               \
        if (e != cudaSuccess) {                                                            \
            printf("%s failed: %s\n", #x, cudaGetErrorString(e));                          \
            return 1;                                                                      \
        }                                                                                  \
    } while (0)

__device__ __forceinline__ uint32_t su32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint32_t b, uint32_t c) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(b), "r"(c));
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(b) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t b, uint32_t par) {
    asm volatile(
        "{\n\t.reg .pred p;\nW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n}" ::"r"(b),
        "r"(par)
        : "memory");
}
__device__ __forceinline__ void tma2d(uint32_t dst, const CUtensorMap *m, uint32_t bar, int c0, int c1) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(
            dst),
        "l"(m), "r"(bar), "r"(c0), "r"(c1)
        : "memory");
}

__device__ __forceinline__ void bulk1d(uint32_t dst, const void *src, uint32_t bytes, uint32_t bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
                 "l"(src), "r"(bytes), "r"(bar)
                 : "memory");
}
// box_rows == 0: one contiguous 16 KB cp.async.bulk per stage (a pre-packed tile), else
// stage = 16 KB = 128 rows x 64 cols, loaded as 128 / box_rows boxes
__global__ void __launch_bounds__(64, 1) stream_kernel(const __grid_constant__ CUtensorMap m, int S, int box_rows,
                                                      int row_blocks_per_cta, int kblocks, int reps, int nrb,
                                                      const uint8_t *base) {
    extern __shared__ __align__(1024) uint8_t raw[];
    uint8_t *sm = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(raw) + 1023) & ~uintptr_t(1023));
    uint64_t *bars = reinterpret_cast<uint64_t *>(sm + S * 16384);
    const uint32_t full0 = su32(bars), empty0 = su32(bars + S);
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) mbar_init(full0 + 8 * s, 1), mbar_init(empty0 + 8 * s, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const int per = row_blocks_per_cta * kblocks, total = per * reps;
    if (threadIdx.x == 0) {
        int s = 0;
        uint32_t ph = 0;
        for (int i = 0; i < total; ++i) {
            mbar_wait(empty0 + 8 * s, ph ^ 1);
            mbar_expect_tx(full0 + 8 * s, 16384);
            const int ii = i % per;
            const int rb = (blockIdx.x * row_blocks_per_cta + ii / kblocks) % nrb, kb = ii % kblocks;
            if (box_rows == 0)
                bulk1d(su32(sm + s * 16384), base + ((long)rb * kblocks + kb) * 16384, 16384, full0 + 8 * s);
            else
                for (int r = 0; r < 128; r += box_rows)
                    tma2d(su32(sm + s * 16384 + r * 128), &m, full0 + 8 * s, kb * 64, rb * 128 + r);
            if (++s == S) s = 0, ph ^= 1;
        }
    } else if (threadIdx.x == 32) {
        int s = 0;
        uint32_t ph = 0;
        for (int i = 0; i < total; ++i) {
            mbar_wait(full0 + 8 * s, ph);
            mbar_arrive(empty0 + 8 * s);
            if (++s == S) s = 0, ph ^= 1;
        }
    }
}

int main() {
    CUresult (*encode)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *, const cuuint64_t *,
                       const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle,
                       CUtensorMapL2promotion, CUtensorMapFloatOOBfill) = nullptr;
    cudaDriverEntryPointQueryResult q;
    CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void **)&encode, cudaEnableDefault, &q));
    const long cols = 1024;  // row pitch 2 KB (an LSTM W[4H][H] with H = 1024)
    const long big_rows = 1L << 17;  // 256 MB > L2
    void *buf;
    CK(cudaMalloc(&buf, big_rows * cols * 2));
    CK(cudaMemset(buf, 0, big_rows * cols * 2));
    CK(cudaFuncSetAttribute(stream_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 12 * 16384 + 2048));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    printf("%6s %4s %4s %8s %10s %10s\n", "grid", "S", "box", "MB", "us", "GB/s");
    for (long rows : {big_rows, 1L << 14}) {  // 256 MB (HBM) and 32 MB (L2-resident, 2nd pass)
        for (int box_rows : {0, 64, 128}) {
            CUtensorMap m;
            cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
            cuuint64_t strides[1] = {(cuuint64_t)cols * 2};
            cuuint32_t box[2] = {64, (cuuint32_t)(box_rows ? box_rows : 64)};
            cuuint32_t es[2] = {1, 1};
            if (encode(&m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, buf, dims, strides, box, es,
                       CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                       CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
                printf("encode failed\n");
                return 1;
            }
            for (int grid : {64, 128, 148}) {
                for (int S : {4, 8}) {
                    const int kblocks = (int)(cols / 64);
                    const int nrb = (int)(rows / 128);
                    const int rbs = nrb / grid > 0 ? nrb / grid : 1;
                    const int reps = rows == big_rows ? 1 : 8;
                    const double mb = (double)grid * rbs * kblocks * reps * 16384 / 1e6;
                    const int smem = S * 16384 + 2048;
                    stream_kernel<<<grid, 64, smem>>>(m, S, box_rows, rbs, kblocks, reps, nrb, (const uint8_t *)buf);  // warm
                    CK(cudaEventRecord(e0));
                    for (int it = 0; it < 3; ++it) stream_kernel<<<grid, 64, smem>>>(m, S, box_rows, rbs, kblocks, reps, nrb, (const uint8_t *)buf);
                    CK(cudaEventRecord(e1));
                    CK(cudaEventSynchronize(e1));
                    float ms;
                    cudaEventElapsedTime(&ms, e0, e1);
                    const double us = ms * 1e3 / 3;
                    printf("%6d %4d %4d %8.1f %10.1f %10.1f %s\n", grid, S, box_rows, mb, us, mb / us * 1e3,
                           rows == big_rows ? "HBM" : "L2");
                }
            }
        }
    }
    return 0;
}
