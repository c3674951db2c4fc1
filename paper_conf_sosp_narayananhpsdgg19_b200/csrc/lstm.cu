// lstm.cu -- LSTM cell (forward / backward-through-time) and embedding kernels.
//
// The LSTM layer (PyTorch form, gates i, f, g, o; h0 = c0 = 0; R22) is run as
//   Gx = X W_ih^T                         one batched tensor-core GEMM over all T*B rows
//   for t: Gh = h_{t-1} W_hh^T            recurrent GEMM (M = B) ...
//          cell(Gx[t] + Gh + b_ih + b_hh) ... fused with this elementwise cell kernel
// and backward as
//   for t = T-1..0: dh = dY[t] + da_{t+1} W_hh;  cell backward -> da_t  (elementwise)
//   dX = da W_ih, dW_ih = da^T X, dW_hh = da[1..]^T h[..T-2], db = sum da   (batched GEMMs)
// so every FLOP-heavy piece is a tensor-core GEMM of the shared kernel; only the
// recurrence-bound elementwise work lives here.
#include <cuda_bf16.h>

#include "pd_internal.h"

namespace pd {
namespace {

__device__ __forceinline__ float ldf(const float *p, long i) { return p[i]; }
__device__ __forceinline__ float ldf(const __nv_bfloat16 *p, long i) { return __bfloat162float(p[i]); }
__device__ __forceinline__ void stf(float *p, long i, float v) { p[i] = v; }
__device__ __forceinline__ void stf(__nv_bfloat16 *p, long i, float v) { p[i] = __float2bfloat16_rn(v); }
__device__ __forceinline__ float sigm(float x) { return 1.0f / (1.0f + __expf(-x)); }

// one thread per (b, j): reads the 4 gate pre-activations of unit j
template <typename T>
__global__ void lstm_cell_fwd_kernel(const float *__restrict__ gx, const float *__restrict__ gh,
                                     const float *__restrict__ b_ih, const float *__restrict__ b_hh,
                                     const float *__restrict__ c_prev, float *__restrict__ gates,
                                     float *__restrict__ c_out, T *__restrict__ h_out, T *__restrict__ y_out, int B,
                                     int H) {
    const long idx = (long)blockIdx.x * blockDim.x + threadIdx.x;
    if (idx >= (long)B * H) return;
    const int b = (int)(idx / H), j = (int)(idx % H);
    float a[4];
#pragma unroll
    for (int g = 0; g < 4; ++g) {
        const long k = (long)b * 4 * H + (long)g * H + j;
        float v = gx[k] + b_ih[g * H + j];
        if (gh) v += gh[k];
        a[g] = v + b_hh[g * H + j];
    }
    const float ig = sigm(a[0]), fg = sigm(a[1]), gg = tanhf(a[2]), og = sigm(a[3]);
    const float cp = c_prev ? c_prev[idx] : 0.f;
    const float c = fg * cp + ig * gg;
    const float h = og * tanhf(c);
    const long k0 = (long)b * 4 * H + j;
    gates[k0] = ig;
    gates[k0 + H] = fg;
    gates[k0 + 2 * H] = gg;
    gates[k0 + 3 * H] = og;
    c_out[idx] = c;
    stf(h_out, idx, h);
    if (y_out) stf(y_out, idx, h);
}

// dh = dy + dh_rec; da (pre-activation gate gradients) and the carried dc
template <typename T>
__global__ void lstm_cell_bwd_kernel(const T *__restrict__ dy, const float *__restrict__ dh_rec,
                                     const float *__restrict__ gates, const float *__restrict__ c,
                                     const float *__restrict__ c_prev, float *__restrict__ dc, T *__restrict__ da,
                                     int B, int H) {
    const long idx = (long)blockIdx.x * blockDim.x + threadIdx.x;
    if (idx >= (long)B * H) return;
    const int b = (int)(idx / H), j = (int)(idx % H);
    const long k0 = (long)b * 4 * H + j;
    const float ig = gates[k0], fg = gates[k0 + H], gg = gates[k0 + 2 * H], og = gates[k0 + 3 * H];
    const float tc = tanhf(c[idx]);
    float dh = ldf(dy, idx);
    if (dh_rec) dh += dh_rec[idx];
    const float dog = dh * tc;
    const float dct = dh * og * (1.f - tc * tc) + dc[idx];
    const float cp = c_prev ? c_prev[idx] : 0.f;
    const float dig = dct * gg, dgg = dct * ig, dfg = dct * cp;
    dc[idx] = dct * fg;
    stf(da, k0, dig * ig * (1.f - ig));
    stf(da, k0 + H, dfg * fg * (1.f - fg));
    stf(da, k0 + 2 * H, dgg * (1.f - gg * gg));
    stf(da, k0 + 3 * H, dog * og * (1.f - og));
}

template <typename T>
__global__ void embedding_fwd_kernel(const int32_t *__restrict__ tok, const T *__restrict__ E, T *__restrict__ y,
                                     long rows, int H) {
    const long stride = (long)gridDim.x * blockDim.x;
    for (long i = (long)blockIdx.x * blockDim.x + threadIdx.x; i < rows * H; i += stride) {
        const long r = i / H;
        y[i] = E[(long)tok[r] * H + (i % H)];
    }
}

// dE[tok[r]] += dy[r] (fp32 atomics; several rows may share a token)
template <typename T>
__global__ void embedding_bwd_kernel(const int32_t *__restrict__ tok, const T *__restrict__ dy, float *__restrict__ dE,
                                     long rows, int H) {
    const long stride = (long)gridDim.x * blockDim.x;
    for (long i = (long)blockIdx.x * blockDim.x + threadIdx.x; i < rows * H; i += stride) {
        const long r = i / H;
        atomicAdd(dE + (long)tok[r] * H + (i % H), ldf(dy, i));
    }
}

unsigned blocks_for(long n) {
    long b = (n + 255) / 256;
    if (b > 148L * 32) b = 148L * 32;
    return (unsigned)(b < 1 ? 1 : b);
}

}  // namespace

cudaError_t lstm_cell_fwd(int bf16, const float *gx, const float *gh, const float *b_ih, const float *b_hh,
                          const float *c_prev, float *gates, float *c_out, void *h_out, void *y_out, int B, int H,
                          cudaStream_t s) {
    const long n = (long)B * H;
    const unsigned blocks = (unsigned)((n + 255) / 256);
    if (bf16)
        lstm_cell_fwd_kernel<<<blocks, 256, 0, s>>>(gx, gh, b_ih, b_hh, c_prev, gates, c_out,
                                                    static_cast<__nv_bfloat16 *>(h_out),
                                                    static_cast<__nv_bfloat16 *>(y_out), B, H);
    else
        lstm_cell_fwd_kernel<<<blocks, 256, 0, s>>>(gx, gh, b_ih, b_hh, c_prev, gates, c_out,
                                                    static_cast<float *>(h_out), static_cast<float *>(y_out), B, H);
    ++tl_launches;
    return cudaGetLastError();
}

cudaError_t lstm_cell_bwd(int bf16, const void *dy, const float *dh_rec, const float *gates, const float *c,
                          const float *c_prev, float *dc, void *da, int B, int H, cudaStream_t s) {
    const long n = (long)B * H;
    const unsigned blocks = (unsigned)((n + 255) / 256);
    if (bf16)
        lstm_cell_bwd_kernel<<<blocks, 256, 0, s>>>(static_cast<const __nv_bfloat16 *>(dy), dh_rec, gates, c, c_prev,
                                                    dc, static_cast<__nv_bfloat16 *>(da), B, H);
    else
        lstm_cell_bwd_kernel<<<blocks, 256, 0, s>>>(static_cast<const float *>(dy), dh_rec, gates, c, c_prev, dc,
                                                    static_cast<float *>(da), B, H);
    ++tl_launches;
    return cudaGetLastError();
}

cudaError_t embedding_fwd(int bf16, const int32_t *tok, const void *E, void *y, long rows, int H, cudaStream_t s) {
    if (bf16)
        embedding_fwd_kernel<<<blocks_for(rows * H), 256, 0, s>>>(tok, static_cast<const __nv_bfloat16 *>(E),
                                                                  static_cast<__nv_bfloat16 *>(y), rows, H);
    else
        embedding_fwd_kernel<<<blocks_for(rows * H), 256, 0, s>>>(tok, static_cast<const float *>(E),
                                                                  static_cast<float *>(y), rows, H);
    ++tl_launches;
    return cudaGetLastError();
}

cudaError_t embedding_bwd(int bf16, const int32_t *tok, const void *dy, float *dE, long rows, int H, cudaStream_t s) {
    if (bf16)
        embedding_bwd_kernel<<<blocks_for(rows * H), 256, 0, s>>>(tok, static_cast<const __nv_bfloat16 *>(dy), dE,
                                                                  rows, H);
    else
        embedding_bwd_kernel<<<blocks_for(rows * H), 256, 0, s>>>(tok, static_cast<const float *>(dy), dE, rows, H);
    ++tl_launches;
    return cudaGetLastError();
}

}  // namespace pd
