// conv.cu -- 3x3 convolution / 2x2 max-pool support kernels on the zero-padded NHWC layout.
//
// Conv and pool activations live on a padded grid [B][H+2][W+2][Cp] (Cp = channels rounded
// up to 8 so every row is 16-byte aligned for TMA) whose halo is always zero: every kernel
// that writes such a buffer writes the halo as 0.  The bf16 path runs convolutions as
// implicit GEMMs on the tensor cores (gemm_tc.cu, ConvGeom: the A-operand rows of each of
// the 9 taps are the same buffer shifted by that tap's pixel offset).  This file holds the
// layout conversion, pooling, the bias reduction over tall gradients, and the fp32 parity
// path's direct convolution kernels.
#include <cuda_bf16.h>

#include <algorithm>

#include "pd_internal.h"

namespace pd {
namespace {

__device__ __forceinline__ float ldf(const float *p, long i) { return p[i]; }
__device__ __forceinline__ float ldf(const __nv_bfloat16 *p, long i) { return __bfloat162float(p[i]); }
__device__ __forceinline__ void stf(float *p, long i, float v) { p[i] = v; }
__device__ __forceinline__ void stf(__nv_bfloat16 *p, long i, float v) { p[i] = __float2bfloat16_rn(v); }

unsigned blocks_for(long n) {
    long b = (n + 255) / 256;
    if (b > 148L * 64) b = 148L * 64;
    return (unsigned)(b < 1 ? 1 : b);
}
#define GRID_STRIDE(i, n) for (long i = (long)blockIdx.x * blockDim.x + threadIdx.x; i < (n); i += (long)gridDim.x * blockDim.x)

// unpadded fp32 NHWC [B][H][W][C] -> padded [B][H+2][W+2][Cp] (halo and channels >= C zero)
template <typename T>
__global__ void pad_nhwc_kernel(const float *__restrict__ in, T *__restrict__ out, int B, int H, int W, int C,
                                int Cp) {
    const int Hp = H + 2, Wp = W + 2;
    const long n = (long)B * Hp * Wp * Cp;
    GRID_STRIDE(i, n) {
        const int c = (int)(i % Cp);
        const long p = i / Cp;
        const int wp = (int)(p % Wp), hp = (int)((p / Wp) % Hp), b = (int)(p / ((long)Wp * Hp));
        float v = 0.f;
        if (c < C && hp >= 1 && hp <= H && wp >= 1 && wp <= W)
            v = in[(((long)b * H + hp - 1) * W + wp - 1) * C + c];
        stf(out, i, v);
    }
}

// 2x2 / stride-2 max-pool.  Input padded [B][H+2][W+2][C]; output padded [B][H/2+2][W/2+2][C]
// (out_padded) or flat [B][H/2][W/2][C].  The first maximum in (dh, dw) order wins ties.
template <typename T>
__global__ void pool_fwd_kernel(const T *__restrict__ x, T *__restrict__ y, int B, int H, int W, int C,
                                int out_padded) {
    const int Ho = H / 2, Wo = W / 2, Hp = H + 2, Wp = W + 2;
    const int Hq = out_padded ? Ho + 2 : Ho, Wq = out_padded ? Wo + 2 : Wo, off = out_padded ? 1 : 0;
    const long n = (long)B * Hq * Wq * C;
    GRID_STRIDE(i, n) {
        const int c = (int)(i % C);
        const long p = i / C;
        const int wq = (int)(p % Wq), hq = (int)((p / Wq) % Hq), b = (int)(p / ((long)Wq * Hq));
        const int ho = hq - off, wo = wq - off;
        float best = 0.f;
        if (ho >= 0 && ho < Ho && wo >= 0 && wo < Wo) {
            bool first = true;
            for (int dh = 0; dh < 2; ++dh)
                for (int dw = 0; dw < 2; ++dw) {
                    const float v = ldf(x, (((long)b * Hp + 2 * ho + dh + 1) * Wp + 2 * wo + dw + 1) * C + c);
                    if (first || v > best) { best = v; first = false; }
                }
        }
        stf(y, i, best);
    }
}

// dX of the pool: each input pixel receives dY of its window iff it is the window's argmax
// (recomputed from the stashed input).  Output padded like the input, halo 0; `mask_relu`
// applies the previous layer's ReLU derivative (x > 0).
template <typename T>
__global__ void pool_bwd_kernel(const T *__restrict__ x, const T *__restrict__ dy, T *__restrict__ dx, int B, int H,
                                int W, int C, int dy_padded, int mask_relu) {
    const int Ho = H / 2, Wo = W / 2, Hp = H + 2, Wp = W + 2;
    const int Hq = dy_padded ? Ho + 2 : Ho, Wq = dy_padded ? Wo + 2 : Wo, off = dy_padded ? 1 : 0;
    const long n = (long)B * Hp * Wp * C;
    GRID_STRIDE(i, n) {
        const int c = (int)(i % C);
        const long p = i / C;
        const int wp = (int)(p % Wp), hp = (int)((p / Wp) % Hp), b = (int)(p / ((long)Wp * Hp));
        float g = 0.f;
        const int h = hp - 1, w = wp - 1;
        if (h >= 0 && h < 2 * Ho && w >= 0 && w < 2 * Wo) {
            const int ho = h / 2, wo = w / 2;
            int arg = -1;
            float best = 0.f;
            for (int dh = 0; dh < 2; ++dh)
                for (int dw = 0; dw < 2; ++dw) {
                    const float v = ldf(x, (((long)b * Hp + 2 * ho + dh + 1) * Wp + 2 * wo + dw + 1) * C + c);
                    if (arg < 0 || v > best) { best = v; arg = dh * 2 + dw; }
                }
            if (arg == (h - 2 * ho) * 2 + (w - 2 * wo)) {
                g = ldf(dy, (((long)b * Hq + ho + off) * Wq + wo + off) * C + c);
                if (mask_relu && !(ldf(x, i) > 0.f)) g = 0.f;
            }
        }
        stf(dx, i, g);
    }
}

// bias gradient over a tall [rows][cols] gradient: block (64-column group, row chunk)
// reduces its chunk and adds it into out (fp32 atomics; out must be zeroed first)
template <typename T>
__global__ void __launch_bounds__(256) col_sum_tall_kernel(const T *__restrict__ G, long rows, int cols,
                                                           long rows_per_block, float *out) {
    __shared__ float part[8][65];
    const int lane = threadIdx.x & 31, rg = threadIdx.x >> 5;
    const long c = (long)blockIdx.x * 64 + 2 * lane;
    const long r0 = (long)blockIdx.y * rows_per_block, r1 = min(rows, r0 + rows_per_block);
    float a0 = 0.f, a1 = 0.f;
    for (long r = r0 + rg; r < r1; r += 8) {
        if (c < cols) a0 += ldf(G, r * cols + c);
        if (c + 1 < cols) a1 += ldf(G, r * cols + c + 1);
    }
    part[rg][2 * lane] = a0;
    part[rg][2 * lane + 1] = a1;
    __syncthreads();
    if (threadIdx.x < 64) {
        const long cc = (long)blockIdx.x * 64 + threadIdx.x;
        if (cc < cols) {
            float g = 0.f;
            for (int q = 0; q < 8; ++q) g += part[q][threadIdx.x];
            atomicAdd(out + cc, g);
        }
    }
}

// bf16, cols % 8 == 0, cols <= 2048: thread = 8 consecutive columns (one 16-byte load) of
// every (256 / (cols/8))-th row of the block's chunk; per-column partials reduced in smem
__global__ void __launch_bounds__(256) col_sum_tall8_kernel(const __nv_bfloat16 *__restrict__ G, long rows,
                                                            int cols, long rows_per_block, float *out) {
    extern __shared__ float red[];  // [256][8]
    const int tpr = cols / 8, rpp = 256 / tpr;  // threads per row, rows per pass
    const int t = threadIdx.x, cg = t % tpr, rr = t / tpr;
    const long r0 = (long)blockIdx.x * rows_per_block, r1 = min(rows, r0 + rows_per_block);
    float a[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
    if (rr < rpp)
        for (long r = r0 + rr; r < r1; r += rpp) {
            const uint4 q = *reinterpret_cast<const uint4 *>(G + r * cols + cg * 8);
            const __nv_bfloat16 *h = reinterpret_cast<const __nv_bfloat16 *>(&q);
#pragma unroll
            for (int i = 0; i < 8; ++i) a[i] += __bfloat162float(h[i]);
        }
#pragma unroll
    for (int i = 0; i < 8; ++i) red[t * 8 + i] = a[i];
    __syncthreads();
    for (int c = t; c < cols; c += 256) {
        const int g = c / 8, i = c % 8;
        float sum = 0.f;
        for (int q = 0; q < rpp; ++q) sum += red[(q * tpr + g) * 8 + i];
        atomicAdd(out + c, sum);
    }
}

// ---------------- fp32 parity path: direct convolutions on the padded layout
// W_dev [Cout][9][Cp] (tap = kh*3 + kw), bias [Cout]
__global__ void conv_fwd_direct_kernel(const float *__restrict__ x, const float *__restrict__ Wd,
                                       const float *__restrict__ bias, float *__restrict__ y, int B, int H, int W,
                                       int Cp, int Cout, int relu) {
    const int Hp = H + 2, Wp = W + 2;
    const long n = (long)B * Hp * Wp * Cout;
    GRID_STRIDE(i, n) {
        const int co = (int)(i % Cout);
        const long p = i / Cout;
        const int wp = (int)(p % Wp), hp = (int)((p / Wp) % Hp);
        float v = 0.f;
        if (hp >= 1 && hp <= H && wp >= 1 && wp <= W) {
            float acc = 0.f;
            for (int kh = 0; kh < 3; ++kh)
                for (int kw = 0; kw < 3; ++kw) {
                    const long q = p + (long)(kh - 1) * Wp + (kw - 1);
                    const float *xr = x + q * Cp;
                    const float *wr = Wd + ((long)co * 9 + kh * 3 + kw) * Cp;
                    for (int ci = 0; ci < Cp; ++ci) acc += xr[ci] * wr[ci];
                }
            v = acc + bias[co];
            if (relu && v < 0.f) v = 0.f;
        }
        y[i] = v;
    }
}

__global__ void conv_dx_direct_kernel(const float *__restrict__ dy, const float *__restrict__ Wd,
                                      const float *__restrict__ xmask, float *__restrict__ dx, int B, int H, int W,
                                      int Cp, int Cout) {
    const int Hp = H + 2, Wp = W + 2;
    const long n = (long)B * Hp * Wp * Cp;
    GRID_STRIDE(i, n) {
        const int ci = (int)(i % Cp);
        const long p = i / Cp;
        const int wp = (int)(p % Wp), hp = (int)((p / Wp) % Hp);
        float v = 0.f;
        if (hp >= 1 && hp <= H && wp >= 1 && wp <= W) {
            float acc = 0.f;
            for (int kh = 0; kh < 3; ++kh)
                for (int kw = 0; kw < 3; ++kw) {
                    const long q = p - (long)(kh - 1) * Wp - (kw - 1);  // output pixel using x[p] via this tap
                    const float *g = dy + q * Cout;
                    for (int co = 0; co < Cout; ++co) acc += g[co] * Wd[((long)co * 9 + kh * 3 + kw) * Cp + ci];
                }
            v = acc;
            if (xmask && !(xmask[i] > 0.f)) v = 0.f;
        }
        dx[i] = v;
    }
}

// dW[co][tap][ci] = sum over interior output pixels p of dy[p][co] * x[p + delta_tap][ci]
__global__ void conv_dw_direct_kernel(const float *__restrict__ dy, const float *__restrict__ x,
                                      float *__restrict__ dW, int B, int H, int W, int Cp, int Cout) {
    const int Hp = H + 2, Wp = W + 2;
    const long n = (long)Cout * 9 * Cp;
    GRID_STRIDE(i, n) {
        const int ci = (int)(i % Cp), tap = (int)((i / Cp) % 9), co = (int)(i / (9L * Cp));
        const int kh = tap / 3, kw = tap % 3;
        float acc = 0.f;
        for (int b = 0; b < B; ++b)
            for (int h = 1; h <= H; ++h)
                for (int w = 1; w <= W; ++w) {
                    const long p = ((long)b * Hp + h) * Wp + w;
                    acc += dy[p * Cout + co] * x[(p + (long)(kh - 1) * Wp + (kw - 1)) * Cp + ci];
                }
        dW[i] = acc;
    }
}

// 8-channel vectorised variants (bf16, C % 8 == 0): one thread = one pooling window x 8
// channels; fwd reads the 4 inputs once, bwd writes all 4 input gradients (no re-reads)
__device__ __forceinline__ void ld8(const __nv_bfloat16 *p, float (&v)[8]) {
    const uint4 r = *reinterpret_cast<const uint4 *>(p);
    const __nv_bfloat16 *h = reinterpret_cast<const __nv_bfloat16 *>(&r);
#pragma unroll
    for (int i = 0; i < 8; ++i) v[i] = __bfloat162float(h[i]);
}
__device__ __forceinline__ void st8(__nv_bfloat16 *p, const float (&v)[8]) {
    uint4 r;
    __nv_bfloat16 *h = reinterpret_cast<__nv_bfloat16 *>(&r);
#pragma unroll
    for (int i = 0; i < 8; ++i) h[i] = __float2bfloat16_rn(v[i]);
    *reinterpret_cast<uint4 *>(p) = r;
}

__global__ void pool_fwd8_kernel(const __nv_bfloat16 *__restrict__ x, __nv_bfloat16 *__restrict__ y, int B, int H,
                                 int W, int C, int out_padded) {
    const int Ho = H / 2, Wo = W / 2, Hp = H + 2, Wp = W + 2, C8 = C / 8;
    const int Hq = out_padded ? Ho + 2 : Ho, Wq = out_padded ? Wo + 2 : Wo, off = out_padded ? 1 : 0;
    const long n = (long)B * Hq * Wq * C8;
    GRID_STRIDE(i, n) {
        const int c8 = (int)(i % C8);
        const long p = i / C8;
        const int wq = (int)(p % Wq), hq = (int)((p / Wq) % Hq), b = (int)(p / ((long)Wq * Hq));
        const int ho = hq - off, wo = wq - off;
        float best[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
        if (ho >= 0 && ho < Ho && wo >= 0 && wo < Wo) {
            for (int dh = 0; dh < 2; ++dh)
                for (int dw = 0; dw < 2; ++dw) {
                    float v[8];
                    ld8(x + (((long)b * Hp + 2 * ho + dh + 1) * Wp + 2 * wo + dw + 1) * C + c8 * 8, v);
#pragma unroll
                    for (int k = 0; k < 8; ++k)
                        if ((dh | dw) == 0 || v[k] > best[k]) best[k] = v[k];
                }
        }
        st8(y + p * C + c8 * 8, best);
    }
}

// one thread per input 2x2 window (and the halo pixels, written as 0)
__global__ void pool_bwd8_kernel(const __nv_bfloat16 *__restrict__ x, const __nv_bfloat16 *__restrict__ dy,
                                 __nv_bfloat16 *__restrict__ dx, int B, int H, int W, int C, int dy_padded,
                                 int mask_relu) {
    const int Ho = H / 2, Wo = W / 2, Hp = H + 2, Wp = W + 2, C8 = C / 8;
    const int Hq = dy_padded ? Ho + 2 : Ho, Wq = dy_padded ? Wo + 2 : Wo, off = dy_padded ? 1 : 0;
    const long nwin = (long)B * Ho * Wo * C8;
    GRID_STRIDE(i, nwin) {
        const int c8 = (int)(i % C8);
        const long p = i / C8;
        const int wo = (int)(p % Wo), ho = (int)((p / Wo) % Ho), b = (int)(p / ((long)Wo * Ho));
        float v[4][8];
        long idx[4];
        for (int q = 0; q < 4; ++q) {
            idx[q] = (((long)b * Hp + 2 * ho + (q >> 1) + 1) * Wp + 2 * wo + (q & 1) + 1) * C + c8 * 8;
            ld8(x + idx[q], v[q]);
        }
        float g[8];
        ld8(dy + (((long)b * Hq + ho + off) * Wq + wo + off) * C + c8 * 8, g);
        float o[4][8];
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            int arg = 0;
            float best = v[0][k];
            for (int q = 1; q < 4; ++q)
                if (v[q][k] > best) { best = v[q][k]; arg = q; }
            for (int q = 0; q < 4; ++q) {
                float gv = q == arg ? g[k] : 0.f;
                if (mask_relu && !(v[q][k] > 0.f)) gv = 0.f;
                o[q][k] = gv;
            }
        }
        for (int q = 0; q < 4; ++q) st8(dx + idx[q], o[q]);
    }
    // halo of dx (and the odd last row/column when H or W is odd: not supported by pd_create)
    const long nh = (long)B * (2 * Wp + 2 * H) * C8;
    GRID_STRIDE(i, nh) {
        const int c8 = (int)(i % C8);
        const long p = i / C8;
        const int per = 2 * Wp + 2 * H, b = (int)(p / per), e = (int)(p % per);
        int hp, wp;
        if (e < Wp) { hp = 0; wp = e; }
        else if (e < 2 * Wp) { hp = Hp - 1; wp = e - Wp; }
        else if (e < 2 * Wp + H) { hp = e - 2 * Wp + 1; wp = 0; }
        else { hp = e - 2 * Wp - H + 1; wp = Wp - 1; }
        const float z[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
        st8(dx + (((long)b * Hp + hp) * Wp + wp) * C + c8 * 8, z);
    }
}

}  // namespace

cudaError_t pad_nhwc(const float *in, void *out, int bf16, int B, int H, int W, int C, int Cp, cudaStream_t s) {
    const long n = (long)B * (H + 2) * (W + 2) * Cp;
    if (bf16) pad_nhwc_kernel<<<blocks_for(n), 256, 0, s>>>(in, static_cast<__nv_bfloat16 *>(out), B, H, W, C, Cp);
    else pad_nhwc_kernel<<<blocks_for(n), 256, 0, s>>>(in, static_cast<float *>(out), B, H, W, C, Cp);
    ++tl_launches;
    return cudaGetLastError();
}

cudaError_t pool_fwd(int bf16, const void *x, void *y, int B, int H, int W, int C, int out_padded, cudaStream_t s) {
    const long n = (long)B * (out_padded ? H / 2 + 2 : H / 2) * (out_padded ? W / 2 + 2 : W / 2) * C;
    if (bf16 && C % 8 == 0) {
        pool_fwd8_kernel<<<blocks_for(n / 8), 256, 0, s>>>(static_cast<const __nv_bfloat16 *>(x),
                                                           static_cast<__nv_bfloat16 *>(y), B, H, W, C, out_padded);
    } else if (bf16)
        pool_fwd_kernel<<<blocks_for(n), 256, 0, s>>>(static_cast<const __nv_bfloat16 *>(x),
                                                      static_cast<__nv_bfloat16 *>(y), B, H, W, C, out_padded);
    else
        pool_fwd_kernel<<<blocks_for(n), 256, 0, s>>>(static_cast<const float *>(x), static_cast<float *>(y), B, H,
                                                      W, C, out_padded);
    ++tl_launches;
    return cudaGetLastError();
}

cudaError_t pool_bwd(int bf16, const void *x, const void *dy, void *dx, int B, int H, int W, int C, int dy_padded,
                     int mask_relu, cudaStream_t s) {
    const long n = (long)B * (H + 2) * (W + 2) * C;
    if (bf16 && C % 8 == 0) {
        pool_bwd8_kernel<<<blocks_for((long)B * (H / 2) * (W / 2) * (C / 8)), 256, 0, s>>>(
            static_cast<const __nv_bfloat16 *>(x), static_cast<const __nv_bfloat16 *>(dy),
            static_cast<__nv_bfloat16 *>(dx), B, H, W, C, dy_padded, mask_relu);
    } else if (bf16)
        pool_bwd_kernel<<<blocks_for(n), 256, 0, s>>>(static_cast<const __nv_bfloat16 *>(x),
                                                      static_cast<const __nv_bfloat16 *>(dy),
                                                      static_cast<__nv_bfloat16 *>(dx), B, H, W, C, dy_padded,
                                                      mask_relu);
    else
        pool_bwd_kernel<<<blocks_for(n), 256, 0, s>>>(static_cast<const float *>(x), static_cast<const float *>(dy),
                                                      static_cast<float *>(dx), B, H, W, C, dy_padded, mask_relu);
    ++tl_launches;
    return cudaGetLastError();
}

cudaError_t col_sum_tall(const void *G, int bf16, long rows, int cols, float *out, cudaStream_t s) {
    if (bf16 && cols % 8 == 0 && cols <= 2048) {
        // ~8 blocks per SM, each reducing a contiguous row chunk
        const long nb = std::max(1L, std::min((rows + 63) / 64, 148L * 8));
        const long rpb8 = (rows + nb - 1) / nb;
        col_sum_tall8_kernel<<<(unsigned)((rows + rpb8 - 1) / rpb8), 256, 256 * 8 * sizeof(float), s>>>(
            static_cast<const __nv_bfloat16 *>(G), rows, cols, rpb8, out);
        ++tl_launches;
        return cudaGetLastError();
    }
    long rpb = 2048;
    long ychunks = (rows + rpb - 1) / rpb;
    if (ychunks > 1024) {
        ychunks = 1024;
        rpb = (rows + ychunks - 1) / ychunks;
    }
    dim3 grid((cols + 63) / 64, (unsigned)ychunks);
    if (bf16)
        col_sum_tall_kernel<<<grid, 256, 0, s>>>(static_cast<const __nv_bfloat16 *>(G), rows, cols, rpb, out);
    else
        col_sum_tall_kernel<<<grid, 256, 0, s>>>(static_cast<const float *>(G), rows, cols, rpb, out);
    ++tl_launches;
    return cudaGetLastError();
}

cudaError_t conv_fwd_f32(const float *x, const float *Wd, const float *bias, float *y, int B, int H, int W, int Cp,
                         int Cout, int relu, cudaStream_t s) {
    const long n = (long)B * (H + 2) * (W + 2) * Cout;
    conv_fwd_direct_kernel<<<blocks_for(n), 256, 0, s>>>(x, Wd, bias, y, B, H, W, Cp, Cout, relu);
    ++tl_launches;
    return cudaGetLastError();
}

cudaError_t conv_dx_f32(const float *dy, const float *Wd, const float *xmask, float *dx, int B, int H, int W, int Cp,
                        int Cout, cudaStream_t s) {
    const long n = (long)B * (H + 2) * (W + 2) * Cp;
    conv_dx_direct_kernel<<<blocks_for(n), 256, 0, s>>>(dy, Wd, xmask, dx, B, H, W, Cp, Cout);
    ++tl_launches;
    return cudaGetLastError();
}

cudaError_t conv_dw_f32(const float *dy, const float *x, float *dW, int B, int H, int W, int Cp, int Cout,
                        cudaStream_t s) {
    const long n = (long)Cout * 9 * Cp;
    conv_dw_direct_kernel<<<blocks_for(n), 256, 0, s>>>(dy, x, dW, B, H, W, Cp, Cout);
    ++tl_launches;
    return cudaGetLastError();
}

}  // namespace pd
