// tma_mc.cu -- per-SM receive bandwidth of TMA unicast vs cluster multicast (tools only; not
// part of the library).  Question: is the ~60-110 GB/s per SM that the GEMM / wavefront
// operands stream at a limit of what an SM can RECEIVE, or of what its TMA unit can ISSUE?
// With .multicast::cluster each CTA of a cluster issues 1/CS of every stage and receives all
// of it; if per-SM received GB/s rises with CS, shared operands (the activation tile every
// item of an LSTM layer reads, the X tile of a small-M GEMM) should be multicast.
//
//   nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a tools/tma_mc.cu -o /tmp/tma_mc -lcuda
//   /tmp/tma_mc
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdint>

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
__device__ __forceinline__ void mbar_wait(uint32_t b, uint32_t par) {
    asm volatile(
        "{\n\t.reg .pred p;\nW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n}" ::"r"(b),
        "r"(par)
        : "memory");
}
__device__ __forceinline__ uint32_t mapa(uint32_t a, uint32_t r) {
    uint32_t o;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(o) : "r"(a), "r"(r));
    return o;
}
__device__ __forceinline__ void arrive_remote(uint32_t bar_cluster) {
    asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(bar_cluster) : "memory");
}
__device__ __forceinline__ void tma2d(uint32_t dst, const CUtensorMap *m, uint32_t bar, int c0, int c1) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(
            dst),
        "l"(m), "r"(bar), "r"(c0), "r"(c1)
        : "memory");
}
__device__ __forceinline__ void tma2d_mc(uint32_t dst, const CUtensorMap *m, uint32_t bar, int c0, int c1,
                                         uint16_t mask) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster [%0], [%1, {%3, "
        "%4}], [%2], %5;" ::"r"(dst),
        "l"(m), "r"(bar), "r"(c0), "r"(c1), "h"(mask)
        : "memory");
}

constexpr int STAGE = 32768;  // 256 rows x 64 bf16 (128 B) per stage
constexpr int NS = 6;

// Each cluster streams `iters` stages of a [rows][64] bf16 matrix region (L2-resident);
// CS = 1: unicast, every CTA loads its whole stage (its own rows); CS > 1: every CTA of the
// cluster receives the SAME stage, loading 256 / CS rows of it with multicast to all.
template <int CS>
__global__ void __launch_bounds__(64, 1) mc_kernel(const __grid_constant__ CUtensorMap m, int iters, int nrb, int box) {
    extern __shared__ __align__(1024) uint8_t raw[];
    uint8_t *sm = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(raw) + 1023) & ~uintptr_t(1023));
    uint64_t *bars = reinterpret_cast<uint64_t *>(sm + NS * STAGE);
    const uint32_t full0 = su32(bars), empty0 = su32(bars + NS);
    uint32_t rank = 0;
    if (CS > 1) asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
    if (threadIdx.x == 0) {
        for (int s = 0; s < NS; ++s) mbar_init(full0 + 8 * s, 1), mbar_init(empty0 + 8 * s, CS);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (CS > 1) {
        asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory");
        asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory");
    } else {
        __syncthreads();
    }
    const int cluster = blockIdx.x / CS;
    if (threadIdx.x == 0) {
        int s = 0;
        uint32_t ph = 0;
        for (int i = 0; i < iters; ++i) {
            mbar_wait(empty0 + 8 * s, ph ^ 1);  // every CTA of the cluster has consumed slot s
            mbar_expect_tx(full0 + 8 * s, STAGE);
            const int rb = (cluster * 7 + i) % nrb;  // 256-row block
            const int rows = 256 / CS;
            for (int r = 0; r < rows; r += box) {
                const int rr = (int)rank * rows + r;
                if (CS == 1)
                    tma2d(su32(sm + s * STAGE + rr * 128), &m, full0 + 8 * s, 0, rb * 256 + rr);
                else
                    tma2d_mc(su32(sm + s * STAGE + rr * 128), &m, full0 + 8 * s, 0, rb * 256 + rr,
                             (uint16_t)((1u << CS) - 1));
            }
            if (++s == NS) s = 0, ph ^= 1;
        }
    } else if (threadIdx.x == 32) {
        int s = 0;
        uint32_t ph = 0;
        for (int i = 0; i < iters; ++i) {
            mbar_wait(full0 + 8 * s, ph);
            for (int q = 0; q < CS; ++q) arrive_remote(mapa(empty0 + 8 * s, q));  // free slot s everywhere
            if (++s == NS) s = 0, ph ^= 1;
        }
    }
    if (CS > 1) {
        asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory");
        asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory");
    }
}

template <int CS>
int run(const CUtensorMap &m, int grid, int nrb, int box, cudaEvent_t e0, cudaEvent_t e1) {
    const int iters = 2048, smem = NS * STAGE + 2048;
    CK(cudaFuncSetAttribute(mc_kernel<CS>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(64);
    cfg.dynamicSmemBytes = smem;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = CS;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    CK(cudaLaunchKernelEx(&cfg, mc_kernel<CS>, m, iters, nrb, box));
    CK(cudaEventRecord(e0));
    for (int it = 0; it < 3; ++it) CK(cudaLaunchKernelEx(&cfg, mc_kernel<CS>, m, iters, nrb, box));
    CK(cudaEventRecord(e1));
    CK(cudaEventSynchronize(e1));
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    const double recv = 3.0 * grid * iters * (double)STAGE;  // bytes received by all SMs
    const double issued = recv / CS;                          // bytes requested from L2
    printf("CS=%d grid=%3d  %8.1f us  received %7.1f GB/s (%5.1f per SM)  L2 reads %7.1f GB/s\n", CS, grid,
           ms * 1e3 / 3, recv / (ms / 1e3) / 1e9, recv / (ms / 1e3) / 1e9 / grid, issued / (ms / 1e3) / 1e9);
    return 0;
}

int main() {
    CUresult (*encode)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *, const cuuint64_t *,
                       const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle,
                       CUtensorMapL2promotion, CUtensorMapFloatOOBfill) = nullptr;
    cudaDriverEntryPointQueryResult q;
    CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void **)&encode, cudaEnableDefault, &q));
    const long rows = 1L << 16;  // 64 x 1024 rows x 128 B = 8 MB: L2-resident
    void *buf;
    CK(cudaMalloc(&buf, rows * 128));
    CK(cudaMemset(buf, 0, rows * 128));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    for (int box_rows : {128, 64}) {
        CUtensorMap m;
        cuuint64_t dims[2] = {64, (cuuint64_t)rows};
        cuuint64_t strides[1] = {128};
        cuuint32_t box[2] = {64, (cuuint32_t)box_rows};
        cuuint32_t es[2] = {1, 1};
        if (encode(&m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, buf, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
            printf("encode failed\n");
            return 1;
        }
        printf("box rows %d (CS=1 loads 256 rows in %d boxes; CS=c loads 256/c rows)\n", box_rows, 256 / box_rows);
        const int nrb = (int)(rows / 256);
        for (int grid : {64, 128, 144}) {
            if (run<1>(m, grid, nrb, box_rows, e0, e1)) return 1;
            if (box_rows == 128 && run<2>(m, grid, nrb, box_rows, e0, e1)) return 1;
            if (box_rows == 64 && run<4>(m, grid, nrb, box_rows, e0, e1)) return 1;
        }
    }
    return 0;
}
