#include <cstdio>
#include <cuda_runtime.h>
__global__ void k(int *c) {
    unsigned r; asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    if (threadIdx.x == 0) atomicAdd(c, 1);
}
int main() {
    int *c; cudaMalloc(&c, 4); cudaMemset(c, 0, 4);
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    for (int grid : {128, 132, 144, 148}) {
        cudaLaunchConfig_t cfg{}; cfg.gridDim = dim3(grid); cfg.blockDim = dim3(256); cfg.dynamicSmemBytes = 200 * 1024;
        cudaLaunchAttribute at[2];
        at[0].id = cudaLaunchAttributeClusterDimension; at[0].val.clusterDim.x = 4; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
        at[1].id = cudaLaunchAttributeCooperative; at[1].val.cooperative = 1;
        cfg.attrs = at; cfg.numAttrs = 2;
        cudaError_t e = cudaLaunchKernelEx(&cfg, k, c);
        cudaError_t e2 = cudaDeviceSynchronize();
        int nc = 0; cudaOccupancyMaxActiveClusters(&nc, (void*)k, &cfg);
        printf("grid %d: launch %s sync %s maxActiveClusters %d\n", grid, cudaGetErrorString(e), cudaGetErrorString(e2), nc);
    }
}
