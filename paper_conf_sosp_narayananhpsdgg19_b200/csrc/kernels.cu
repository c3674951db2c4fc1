// kernels.cu -- fp32 SIMT GEMM (parity path), softmax cross-entropy, bias-gradient column
// sums, optimizer updates that write the next weight version, casts, and the cross-process
// flag signal.  The bf16 tensor-core GEMM lives in gemm_tc.cu.
#include <cuda_bf16.h>

#include "pd_internal.h"

namespace pd {

thread_local uint64_t tl_launches = 0;

namespace {

__device__ __forceinline__ float ld_as_f32(const float *p, long i) { return p[i]; }
__device__ __forceinline__ float ld_as_f32(const __nv_bfloat16 *p, long i) { return __bfloat162float(p[i]); }

// ------------------------------------------------------------------ fp32 SIMT GEMM
// 64x64 output tile per 256-thread block, 4x4 per thread, BK = 16, generic operand
// strides (handles the K-/MN-major views of fwd, dX and dW without transposes).
constexpr int SB_M = 64, SB_N = 64, SB_K = 16;

__global__ void __launch_bounds__(256) sgemm_kernel(Gemm g) {
    __shared__ float As[SB_K][SB_M + 4];
    __shared__ float Bs[SB_K][SB_N + 4];
    const float *A = static_cast<const float *>(g.A);
    const float *B = static_cast<const float *>(g.B);
    const int tid = threadIdx.x;
    const int m0 = blockIdx.y * SB_M, n0 = blockIdx.x * SB_N;
    const int tm = (tid / 16) * 4, tn = (tid % 16) * 4;
    float acc[4][4] = {};
    for (int k0 = 0; k0 < g.K; k0 += SB_K) {
        // 1024 elements of each operand tile, 4 per thread; the fastest index follows the
        // operand's contiguous dimension so global reads coalesce.
        for (int e = tid; e < SB_M * SB_K; e += 256) {
            int mm, kk;
            if (g.amaj == KMAJ) { kk = e % SB_K; mm = e / SB_K; } else { mm = e % SB_M; kk = e / SB_M; }
            const int m = m0 + mm, k = k0 + kk;
            float v = 0.f;
            if (m < g.M && k < g.K) v = g.amaj == KMAJ ? A[(long)m * g.lda + k] : A[(long)k * g.lda + m];
            As[kk][mm] = v;
        }
        for (int e = tid; e < SB_N * SB_K; e += 256) {
            int nn, kk;
            if (g.bmaj == KMAJ) { kk = e % SB_K; nn = e / SB_K; } else { nn = e % SB_N; kk = e / SB_N; }
            const int n = n0 + nn, k = k0 + kk;
            float v = 0.f;
            if (n < g.N && k < g.K) v = g.bmaj == KMAJ ? B[(long)n * g.ldb + k] : B[(long)k * g.ldb + n];
            Bs[kk][nn] = v;
        }
        __syncthreads();
#pragma unroll
        for (int kk = 0; kk < SB_K; ++kk) {
            float a[4], b[4];
#pragma unroll
            for (int i = 0; i < 4; ++i) a[i] = As[kk][tm + i];
#pragma unroll
            for (int i = 0; i < 4; ++i) b[i] = Bs[kk][tn + i];
#pragma unroll
            for (int i = 0; i < 4; ++i)
#pragma unroll
                for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
        }
        __syncthreads();
    }
    float *out = static_cast<float *>(g.out);
    const float *mask = static_cast<const float *>(g.mask);
#pragma unroll
    for (int i = 0; i < 4; ++i) {
        const int m = m0 + tm + i;
        if (m >= g.M) continue;
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const int n = n0 + tn + j;
            if (n >= g.N) continue;
            float v = acc[i][j];
            if (g.epi == EPI_STORE) {
                if (g.bias) v += g.bias[n];
                if (g.relu && v < 0.f) v = 0.f;
            } else if (g.epi == EPI_MASK) {
                if (mask && !(mask[(long)m * g.ldm + n] > 0.f)) v = 0.f;
            }
            out[(long)m * g.ldo + n] = v;
        }
    }
}

// ------------------------------------------------------------------ column sums (bias grads)
// out[c] = sum_r G[r][c]; one thread per column, rows in order (deterministic).
template <typename T>
__global__ void col_sum_kernel(const T *G, long rows, long cols, float *out) {
    const long c = (long)blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= cols) return;
    float acc = 0.f;
    for (long r = 0; r < rows; ++r) acc += ld_as_f32(G, r * cols + c);
    out[c] = acc;
}

// ------------------------------------------------------------------ bias gradient (+ update)
// db[c] = sum_r G[r][c].  A 1024-thread block covers 64 columns (a lane reads 2 adjacent
// columns, so a warp reads one 128-byte row segment) x 32 row groups; each thread sums its
// rows with 8 independent loads in flight, then the 32 partials are added in a fixed order
// (deterministic).  When `master` is given the optimizer update of the bias is applied in
// the same kernel (bf16 path, unreplicated stage); otherwise db is written to grad_out.
template <typename T>
__device__ __forceinline__ float2 ld2_as_f32(const T *p, long i) {
    if constexpr (sizeof(T) == 4) return make_float2(p[i], p[i + 1]);
    else {
        const __nv_bfloat162 h = *reinterpret_cast<const __nv_bfloat162 *>(p + i);
        return __bfloat1622float2(h);
    }
}

template <typename T>
__global__ void __launch_bounds__(1024) bias_grad_kernel(const T *__restrict__ G, long rows, long cols,
                                                         float *grad_out, float *master, __nv_bfloat16 *slot, int opt,
                                                         float *m, float *v, float lr, float b1, float b2, float eps,
                                                         float bc1, float bc2) {
    __shared__ float part[32][65];
    const int lane = threadIdx.x & 31, rg = threadIdx.x >> 5;
    const long c = (long)blockIdx.x * 64 + 2 * lane;
    float a0 = 0.f, a1 = 0.f;
    if (c + 1 < cols) {
        long r = rg;
        for (; r + 7 * 32 < rows; r += 8 * 32) {
            float2 x[8];
#pragma unroll
            for (int u = 0; u < 8; ++u) x[u] = ld2_as_f32(G, (r + u * 32) * cols + c);
#pragma unroll
            for (int u = 0; u < 8; ++u) { a0 += x[u].x; a1 += x[u].y; }
        }
        for (; r < rows; r += 32) {
            const float2 x = ld2_as_f32(G, r * cols + c);
            a0 += x.x;
            a1 += x.y;
        }
    } else if (c < cols) {
        for (long r = rg; r < rows; r += 32) a0 += ld_as_f32(G, r * cols + c);
    }
    part[rg][2 * lane] = a0;
    part[rg][2 * lane + 1] = a1;
    __syncthreads();
    if (threadIdx.x < 64) {
        const long cc = (long)blockIdx.x * 64 + threadIdx.x;
        if (cc >= cols) return;
        float g = part[0][threadIdx.x];
        for (int q = 1; q < 32; ++q) g += part[q][threadIdx.x];
        if (grad_out) grad_out[cc] = g;
        if (master) {
            float w = master[cc];
            if (opt == PD_SGD) {
                w = w - lr * g;
            } else {
                const float mm = b1 * m[cc] + (1.f - b1) * g;
                const float vv = b2 * v[cc] + (1.f - b2) * g * g;
                m[cc] = mm;
                v[cc] = vv;
                w = w - lr * (mm / bc1) / (sqrtf(vv / bc2) + eps);
            }
            master[cc] = w;
            if (slot) slot[cc] = __float2bfloat16_rn(w);
        }
    }
}

// Tall G (rows >= 1024, e.g. LSTM da over T*B rows): the rows are split over a cluster of CS
// CTAs (grid.y), so 4x more SMs stream G; each CTA reduces its rows as above, then rank 0
// adds the CS partial sums through distributed shared memory in rank order (deterministic)
// and applies the update.
template <typename T, int CS>
__global__ void __launch_bounds__(1024) bias_grad_cluster_kernel(const T *__restrict__ G, long rows, long cols,
                                                                 float *grad_out, float *master,
                                                                 __nv_bfloat16 *slot, int opt, float *m, float *v,
                                                                 float lr, float b1, float b2, float eps, float bc1,
                                                                 float bc2) {
    __shared__ float part[32][65];
    __shared__ float psum[64];
    const int lane = threadIdx.x & 31, rg = threadIdx.x >> 5;
    uint32_t crank;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(crank));
    const long r_lo = rows * (long)crank / CS, r_hi = rows * (long)(crank + 1) / CS;
    const long c = (long)blockIdx.x * 64 + 2 * lane;
    float a0 = 0.f, a1 = 0.f;
    if (c + 1 < cols) {
        long r = r_lo + rg;
        for (; r + 7 * 32 < r_hi; r += 8 * 32) {
            float2 x[8];
#pragma unroll
            for (int u = 0; u < 8; ++u) x[u] = ld2_as_f32(G, (r + u * 32) * cols + c);
#pragma unroll
            for (int u = 0; u < 8; ++u) { a0 += x[u].x; a1 += x[u].y; }
        }
        for (; r < r_hi; r += 32) {
            const float2 x = ld2_as_f32(G, r * cols + c);
            a0 += x.x;
            a1 += x.y;
        }
    } else if (c < cols) {
        for (long r = r_lo + rg; r < r_hi; r += 32) a0 += ld_as_f32(G, r * cols + c);
    }
    part[rg][2 * lane] = a0;
    part[rg][2 * lane + 1] = a1;
    __syncthreads();
    if (threadIdx.x < 64) {
        float g = part[0][threadIdx.x];
        for (int q = 1; q < 32; ++q) g += part[q][threadIdx.x];
        psum[threadIdx.x] = g;
    }
    asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    if (crank == 0 && threadIdx.x < 64) {
        const long cc = (long)blockIdx.x * 64 + threadIdx.x;
        if (cc < cols) {
            const uint32_t local = (uint32_t)__cvta_generic_to_shared(&psum[threadIdx.x]);
            float g = 0.f;
#pragma unroll
            for (int q = 0; q < CS; ++q) {
                uint32_t ra;
                float x;
                asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(local), "r"((uint32_t)q));
                asm volatile("ld.shared::cluster.f32 %0, [%1];" : "=f"(x) : "r"(ra) : "memory");
                g += x;
            }
            if (grad_out) grad_out[cc] = g;
            if (master) {
                float w = master[cc];
                if (opt == PD_SGD) {
                    w = w - lr * g;
                } else {
                    const float mm = b1 * m[cc] + (1.f - b1) * g;
                    const float vv = b2 * v[cc] + (1.f - b2) * g * g;
                    m[cc] = mm;
                    v[cc] = vv;
                    w = w - lr * (mm / bc1) / (sqrtf(vv / bc2) + eps);
                }
                master[cc] = w;
                if (slot) slot[cc] = __float2bfloat16_rn(w);
            }
        }
    }
    // no CTA may exit while rank 0 still reads its partial sums
    asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// ------------------------------------------------------------------ softmax cross-entropy
// One block per row: max, sum of exp, loss += (lse - z[label]) / rows, and
// dlogits = (softmax - onehot) / rows written in the logits' dtype (L1217, R8).
template <typename T>
__global__ void __launch_bounds__(256) softmax_ce_kernel(const T *z, const int32_t *labels, long rows, int C, T *dz,
                                                         float *loss) {
    const long r = blockIdx.x;
    const T *zr = z + r * C;
    __shared__ float red[32];
    float m = -INFINITY;
    for (int c = threadIdx.x; c < C; c += blockDim.x) m = fmaxf(m, ld_as_f32(zr, c));
    for (int o = 16; o; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = m;
    __syncthreads();
    if (threadIdx.x < 32) {
        float v = threadIdx.x < (blockDim.x >> 5) ? red[threadIdx.x] : -INFINITY;
        for (int o = 16; o; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
        if (threadIdx.x == 0) red[0] = v;
    }
    __syncthreads();
    m = red[0];
    __syncthreads();
    float s = 0.f;
    for (int c = threadIdx.x; c < C; c += blockDim.x) s += __expf(ld_as_f32(zr, c) - m);
    for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x < 32) {
        float v = threadIdx.x < (blockDim.x >> 5) ? red[threadIdx.x] : 0.f;
        for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        if (threadIdx.x == 0) red[0] = v;
    }
    __syncthreads();
    s = red[0];
    const int lab = labels[r];
    const float inv_rows = 1.0f / (float)rows;
    const float inv_s = 1.0f / s;
    for (int c = threadIdx.x; c < C; c += blockDim.x) {
        const float p = __expf(ld_as_f32(zr, c) - m) * inv_s;
        const float d = (p - (c == lab ? 1.f : 0.f)) * inv_rows;
        if constexpr (sizeof(T) == 4) dz[r * C + c] = d;
        else dz[r * C + c] = __float2bfloat16_rn(d);
    }
    if (threadIdx.x == 0) atomicAdd(loss, (m + __logf(s) - ld_as_f32(zr, lab)) * inv_rows);
}

// bf16 rows with C % 8 == 0 (16-byte aligned) and C <= 32 * blockDim.x: the row is read from
// HBM ONCE into registers (up to 4 x 8 bf16 per thread, 16-byte loads), max / sum-of-exp are
// block reductions over the registers, and dlogits is written with 16-byte stores -- one read
// and one write of the logits (HBM-bound: 4 B per logit)
__device__ __forceinline__ float block_reduce(float v, float *red, bool is_max) {
    for (int o = 16; o; o >>= 1) {
        const float u = __shfl_xor_sync(0xffffffffu, v, o);
        v = is_max ? fmaxf(v, u) : v + u;
    }
    __syncthreads();  // red[] free (previous reduction consumed)
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = v;
    __syncthreads();
    const int nw = blockDim.x >> 5;
    v = (int)(threadIdx.x & 31) < nw ? red[threadIdx.x & 31] : (is_max ? -INFINITY : 0.f);
    for (int o = 16; o; o >>= 1) {
        const float u = __shfl_xor_sync(0xffffffffu, v, o);
        v = is_max ? fmaxf(v, u) : v + u;
    }
    return v;
}

__global__ void __launch_bounds__(1024) softmax_ce_bf16_row_kernel(const __nv_bfloat16 *__restrict__ z,
                                                                   const int32_t *__restrict__ labels, long rows,
                                                                   int C, __nv_bfloat16 *__restrict__ dz,
                                                                   float *loss) {
    constexpr int KMAX = 4;
    const long r = blockIdx.x;
    const uint4 *zr = reinterpret_cast<const uint4 *>(z + r * C);
    uint4 *dr = reinterpret_cast<uint4 *>(dz + r * C);
    const int n8 = C / 8;
    __shared__ float red[32];
    uint4 raw[KMAX];
    float m = -INFINITY;
#pragma unroll
    for (int k = 0; k < KMAX; ++k) {
        const int i = threadIdx.x + k * blockDim.x;
        if (i < n8) {
            raw[k] = zr[i];
            const __nv_bfloat16 *h = reinterpret_cast<const __nv_bfloat16 *>(&raw[k]);
#pragma unroll
            for (int j = 0; j < 8; ++j) m = fmaxf(m, __bfloat162float(h[j]));
        }
    }
    m = block_reduce(m, red, true);
    float s = 0.f;
#pragma unroll
    for (int k = 0; k < KMAX; ++k) {
        const int i = threadIdx.x + k * blockDim.x;
        if (i < n8) {
            const __nv_bfloat16 *h = reinterpret_cast<const __nv_bfloat16 *>(&raw[k]);
#pragma unroll
            for (int j = 0; j < 8; ++j) s += __expf(__bfloat162float(h[j]) - m);
        }
    }
    s = block_reduce(s, red, false);
    const int lab = labels[r];
    const float inv_rows = 1.0f / (float)rows;
    const float inv_s = 1.0f / s;
#pragma unroll
    for (int k = 0; k < KMAX; ++k) {
        const int i = threadIdx.x + k * blockDim.x;
        if (i < n8) {
            const __nv_bfloat16 *h = reinterpret_cast<const __nv_bfloat16 *>(&raw[k]);
            uint4 o;
            uint32_t *ow = reinterpret_cast<uint32_t *>(&o);
#pragma unroll
            for (int j = 0; j < 8; j += 2) {
                const int c = i * 8 + j;
                const float d0 = (__expf(__bfloat162float(h[j]) - m) * inv_s - (c == lab ? 1.f : 0.f)) * inv_rows;
                const float d1 = (__expf(__bfloat162float(h[j + 1]) - m) * inv_s - (c + 1 == lab ? 1.f : 0.f)) * inv_rows;
                __nv_bfloat162 p2 = __floats2bfloat162_rn(d0, d1);
                ow[j / 2] = *reinterpret_cast<uint32_t *>(&p2);
            }
            dr[i] = o;
        }
    }
    if (threadIdx.x == 0) atomicAdd(loss, (m + __logf(s) - __bfloat162float(z[r * C + lab])) * inv_rows);
}

// ------------------------------------------------------------------ optimizer updates
__global__ void sgd_f32_kernel(const float *__restrict__ in, const float *__restrict__ g, float *__restrict__ out,
                               long n, float lr) {
    const long stride = (long)gridDim.x * blockDim.x;
    long i = (long)blockIdx.x * blockDim.x + threadIdx.x;
    if ((n & 3) == 0 && (((uintptr_t)in | (uintptr_t)g | (uintptr_t)out) & 15) == 0) {
        const long n4 = n >> 2;
        for (; i < n4; i += stride) {
            float4 w = reinterpret_cast<const float4 *>(in)[i], d = reinterpret_cast<const float4 *>(g)[i];
            w.x -= lr * d.x; w.y -= lr * d.y; w.z -= lr * d.z; w.w -= lr * d.w;
            reinterpret_cast<float4 *>(out)[i] = w;
        }
        return;
    }
    for (; i < n; i += stride) out[i] = in[i] - lr * g[i];
}

__device__ __forceinline__ float adam_step(float w, float g, float &m, float &v, float lr, float b1, float b2,
                                           float eps, float bc1, float bc2) {
    m = b1 * m + (1.f - b1) * g;
    v = b2 * v + (1.f - b2) * g * g;
    const float mh = m / bc1, vh = v / bc2;
    return w - lr * mh / (sqrtf(vh) + eps);
}

__global__ void adam_f32_kernel(const float *in, const float *g, float *out, float *m, float *v, long n, float lr,
                                float b1, float b2, float eps, float bc1, float bc2) {
    const long stride = (long)gridDim.x * blockDim.x;
    for (long i = (long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        float mm = m[i], vv = v[i];
        out[i] = adam_step(in[i], g[i], mm, vv, lr, b1, b2, eps, bc1, bc2);
        m[i] = mm;
        v[i] = vv;
    }
}

// master -= update(mean over replicas of grads); slot = bf16(master) (or fp32 slot)
__global__ void update_master_kernel(float *master, __nv_bfloat16 *slot_bf16, float *slot_f32,
                                     const float *const *grads, int R, long goff, long n, int opt, float *m, float *v,
                                     float lr, float b1, float b2, float eps, float bc1, float bc2) {
    const long stride = (long)gridDim.x * blockDim.x;
    const float invR = 1.0f / (float)R;
    for (long i = (long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        float g = 0.f;
        for (int r = 0; r < R; ++r) g += grads[r][goff + i];  // replica order (R7)
        if (R > 1) g = g * invR;
        float w = master[i];
        if (opt == PD_SGD) {
            w = w - lr * g;
        } else {
            float mm = m[i], vv = v[i];
            w = adam_step(w, g, mm, vv, lr, b1, b2, eps, bc1, bc2);
            m[i] = mm;
            v[i] = vv;
        }
        master[i] = w;
        if (slot_bf16) slot_bf16[i] = __float2bfloat16_rn(w);
        if (slot_f32) slot_f32[i] = w;
    }
}

// one unreplicated gradient g (fp32, 16-byte aligned, n % 4 == 0): master -= SGD/Adam step,
// slot = bf16(master); 4 elements per thread, 16-byte loads/stores (HBM-bound: SGD 14 B,
// Adam 30 B per parameter: g 4, master 4 + 4, m and v 8 + 8, slot 2)
template <bool ADAM>
__global__ void __launch_bounds__(256) update_vec4_kernel(float *__restrict__ master, __nv_bfloat16 *__restrict__ slot,
                                                          const float *__restrict__ g, long n4, float *__restrict__ m,
                                                          float *__restrict__ v, float lr, float b1, float b2,
                                                          float eps, float bc1, float bc2) {
    const long stride = (long)gridDim.x * blockDim.x;
    for (long i = (long)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += stride) {
        const float4 gg = reinterpret_cast<const float4 *>(g)[i];
        float4 w = reinterpret_cast<const float4 *>(master)[i];
        if constexpr (ADAM) {
            float4 mm = reinterpret_cast<const float4 *>(m)[i], vv = reinterpret_cast<const float4 *>(v)[i];
            w.x = adam_step(w.x, gg.x, mm.x, vv.x, lr, b1, b2, eps, bc1, bc2);
            w.y = adam_step(w.y, gg.y, mm.y, vv.y, lr, b1, b2, eps, bc1, bc2);
            w.z = adam_step(w.z, gg.z, mm.z, vv.z, lr, b1, b2, eps, bc1, bc2);
            w.w = adam_step(w.w, gg.w, mm.w, vv.w, lr, b1, b2, eps, bc1, bc2);
            reinterpret_cast<float4 *>(m)[i] = mm;
            reinterpret_cast<float4 *>(v)[i] = vv;
        } else {
            w.x -= lr * gg.x;
            w.y -= lr * gg.y;
            w.z -= lr * gg.z;
            w.w -= lr * gg.w;
        }
        reinterpret_cast<float4 *>(master)[i] = w;
        __nv_bfloat162 lo = __floats2bfloat162_rn(w.x, w.y), hi = __floats2bfloat162_rn(w.z, w.w);
        uint2 o;
        o.x = *reinterpret_cast<uint32_t *>(&lo);
        o.y = *reinterpret_cast<uint32_t *>(&hi);
        reinterpret_cast<uint2 *>(slot)[i] = o;
    }
}

__global__ void f32_to_bf16_kernel(const float *in, __nv_bfloat16 *out, long n) {
    const long stride = (long)gridDim.x * blockDim.x;
    long i = (long)blockIdx.x * blockDim.x + threadIdx.x;
    if ((n & 3) == 0 && ((uintptr_t)in & 15) == 0 && ((uintptr_t)out & 7) == 0) {
        for (; i < n / 4; i += stride) {
            const float4 x = reinterpret_cast<const float4 *>(in)[i];
            __nv_bfloat162 lo = __floats2bfloat162_rn(x.x, x.y), hi = __floats2bfloat162_rn(x.z, x.w);
            uint2 o;
            o.x = *reinterpret_cast<uint32_t *>(&lo);
            o.y = *reinterpret_cast<uint32_t *>(&hi);
            reinterpret_cast<uint2 *>(out)[i] = o;
        }
        return;
    }
    for (; i < n; i += stride) out[i] = __float2bfloat16_rn(in[i]);
}
__global__ void bf16_to_f32_kernel(const __nv_bfloat16 *in, float *out, long n) {
    const long stride = (long)gridDim.x * blockDim.x;
    for (long i = (long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) out[i] = __bfloat162float(in[i]);
}

// Release-store of a monotonically increasing counter into (possibly peer-mapped) memory.
// Stream order makes every earlier kernel's writes complete before this kernel runs; the
// system-scope fence orders them before the flag for the observing GPU.
__global__ void signal_kernel(uint32_t *flag, uint32_t value) {
    __threadfence_system();
    asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(flag), "r"(value) : "memory");
}

int grid_for(long n, int block = 256) {
    long b = (n + block - 1) / block;
    if (b > 148L * 16) b = 148L * 16;  // grid-stride beyond 16 waves of the 148 SMs
    return (int)(b < 1 ? 1 : b);
}

}  // namespace

cudaError_t gemm_f32(const Gemm &g, cudaStream_t s) {
    if (g.epi != EPI_STORE && g.epi != EPI_MASK && g.epi != EPI_F32) return cudaErrorInvalidValue;
    dim3 grid((g.N + SB_N - 1) / SB_N, (g.M + SB_M - 1) / SB_M);
    sgemm_kernel<<<grid, 256, 0, s>>>(g);
    ++tl_launches;
    return cudaGetLastError();
}

cudaError_t col_sum(const void *G, int bf16, long rows, long cols, float *out, cudaStream_t s) {
    const int blocks = (int)((cols + 255) / 256);
    if (bf16) col_sum_kernel<<<blocks, 256, 0, s>>>(static_cast<const __nv_bfloat16 *>(G), rows, cols, out);
    else col_sum_kernel<<<blocks, 256, 0, s>>>(static_cast<const float *>(G), rows, cols, out);
    ++tl_launches;
    return cudaGetLastError();
}

cudaError_t bias_grad(const void *G, int bf16, long rows, long cols, float *grad_out, float *master,
                      __nv_bfloat16 *slot, int opt, float *m, float *v, float lr, float b1, float b2, float eps,
                      int step, cudaStream_t s) {
    const float bc1 = 1.f - powf(b1, (float)step), bc2 = 1.f - powf(b2, (float)step);
    const unsigned blocks = (unsigned)((cols + 63) / 64);
    if (rows >= 1024) {
        constexpr int CS = 4;
        cudaLaunchConfig_t cfg{};
        cfg.gridDim = dim3(blocks, CS);
        cfg.blockDim = dim3(1024);
        cfg.stream = s;
        cudaLaunchAttribute attr[1];
        attr[0].id = cudaLaunchAttributeClusterDimension;
        attr[0].val.clusterDim.x = 1;
        attr[0].val.clusterDim.y = CS;
        attr[0].val.clusterDim.z = 1;
        cfg.attrs = attr;
        cfg.numAttrs = 1;
        ++tl_launches;
        if (bf16)
            return cudaLaunchKernelEx(&cfg, bias_grad_cluster_kernel<__nv_bfloat16, CS>,
                                      static_cast<const __nv_bfloat16 *>(G), rows, cols, grad_out, master, slot, opt,
                                      m, v, lr, b1, b2, eps, bc1, bc2);
        return cudaLaunchKernelEx(&cfg, bias_grad_cluster_kernel<float, CS>, static_cast<const float *>(G), rows, cols,
                                  grad_out, master, slot, opt, m, v, lr, b1, b2, eps, bc1, bc2);
    }
    if (bf16)
        bias_grad_kernel<<<blocks, 1024, 0, s>>>(static_cast<const __nv_bfloat16 *>(G), rows, cols, grad_out, master,
                                                 slot, opt, m, v, lr, b1, b2, eps, bc1, bc2);
    else
        bias_grad_kernel<<<blocks, 1024, 0, s>>>(static_cast<const float *>(G), rows, cols, grad_out, master, slot,
                                                 opt, m, v, lr, b1, b2, eps, bc1, bc2);
    ++tl_launches;
    return cudaGetLastError();
}

cudaError_t softmax_ce(const void *logits, int bf16, const int32_t *labels, long rows, int C, void *dlogits,
                       float *loss_out, cudaStream_t s) {
    if (bf16 && C % 8 == 0 && C <= 32 * 1024 && ((uintptr_t)logits & 15) == 0 && ((uintptr_t)dlogits & 15) == 0) {
        const int n8 = C / 8;
        int threads = ((n8 + 3) / 4 + 31) / 32 * 32;  // <= 4 chunks of 8 per thread
        if (threads < 64) threads = 64;
        softmax_ce_bf16_row_kernel<<<(unsigned)rows, threads, 0, s>>>(static_cast<const __nv_bfloat16 *>(logits),
                                                                      labels, rows, C,
                                                                      static_cast<__nv_bfloat16 *>(dlogits), loss_out);
    } else if (bf16)
        softmax_ce_kernel<<<(unsigned)rows, 256, 0, s>>>(static_cast<const __nv_bfloat16 *>(logits), labels, rows, C,
                                                         static_cast<__nv_bfloat16 *>(dlogits), loss_out);
    else
        softmax_ce_kernel<<<(unsigned)rows, 256, 0, s>>>(static_cast<const float *>(logits), labels, rows, C,
                                                         static_cast<float *>(dlogits), loss_out);
    ++tl_launches;
    return cudaGetLastError();
}

cudaError_t sgd_f32(const float *in, const float *g, float *out, long n, float lr, cudaStream_t s) {
    sgd_f32_kernel<<<grid_for(n / 4 + 1), 256, 0, s>>>(in, g, out, n, lr);
    ++tl_launches;
    return cudaGetLastError();
}

cudaError_t adam_f32(const float *in, const float *g, float *out, float *m, float *v, long n, float lr, float b1,
                     float b2, float eps, int step, cudaStream_t s) {
    const float bc1 = 1.f - powf(b1, (float)step), bc2 = 1.f - powf(b2, (float)step);
    adam_f32_kernel<<<grid_for(n), 256, 0, s>>>(in, g, out, m, v, n, lr, b1, b2, eps, bc1, bc2);
    ++tl_launches;
    return cudaGetLastError();
}

cudaError_t update_master(float *master, __nv_bfloat16 *slot_bf16, float *slot_f32, const float *const *grads,
                          int R, long goff, long n, int opt, float *m, float *v, float lr, float b1, float b2,
                          float eps, int step, cudaStream_t s) {
    const float bc1 = 1.f - powf(b1, (float)step), bc2 = 1.f - powf(b2, (float)step);
    update_master_kernel<<<grid_for(n), 256, 0, s>>>(master, slot_bf16, slot_f32, grads, R, goff, n, opt, m, v, lr,
                                                     b1, b2, eps, bc1, bc2);
    ++tl_launches;
    return cudaGetLastError();
}

// (GPipe flush update: the same kernel with R = D gradient buffers of one worker -- the
// group's gradients summed in t order, times 1/D -- and nout = 1 destination.)
//
// Replica sync of one round, sharded (reduce-scatter -> update -> all-gather through peer
// memory): this replica owns parameters [lo, hi) (16-byte multiples).  For each of them it
// sums the R replicas' fp32 gradients in replica order (R7) over NVLink peer loads, applies
// the optimizer to its own weights w_in (fp32 master on the bf16 path, the latest fp32 slot
// on the fp32 path) and Adam state, and stores the new version into EVERY replica: fp32 into
// out_f32[q] (masters / fp32 slots), bf16 into out_bf16[q] (bf16 slots).  Per replica and
// round: (R-1)/R * 4 B/param of peer reads, (R-1)/R * (4 [+ 2]) B/param of peer stores,
// instead of (R-1) * 4 B/param of reads and a redundant full update on every replica.
template <bool ADAM>
__global__ void __launch_bounds__(256) update_shard_kernel(const float *const *__restrict__ grads, int R, long lo,
                                                           long n4, const float *w_in, float *const *__restrict__ out_f32,
                                                           __nv_bfloat16 *const *__restrict__ out_bf16, int nout,
                                                           float *__restrict__ m, float *__restrict__ v, float lr,
                                                           float b1, float b2, float eps, float bc1, float bc2) {
    const float invR = 1.0f / (float)R;
    const long stride = (long)gridDim.x * blockDim.x;
    for (long k = (long)blockIdx.x * blockDim.x + threadIdx.x; k < n4; k += stride) {
        const long i = lo + 4 * k;
        float4 g = *reinterpret_cast<const float4 *>(grads[0] + i);
        for (int r = 1; r < R; ++r) {  // replica order
            const float4 x = *reinterpret_cast<const float4 *>(grads[r] + i);
            g.x += x.x, g.y += x.y, g.z += x.z, g.w += x.w;
        }
        if (R > 1) g.x *= invR, g.y *= invR, g.z *= invR, g.w *= invR;
        float4 w = *reinterpret_cast<const float4 *>(w_in + i);
        if constexpr (ADAM) {
            float4 mm = *reinterpret_cast<const float4 *>(m + i), vv = *reinterpret_cast<const float4 *>(v + i);
            w.x = adam_step(w.x, g.x, mm.x, vv.x, lr, b1, b2, eps, bc1, bc2);
            w.y = adam_step(w.y, g.y, mm.y, vv.y, lr, b1, b2, eps, bc1, bc2);
            w.z = adam_step(w.z, g.z, mm.z, vv.z, lr, b1, b2, eps, bc1, bc2);
            w.w = adam_step(w.w, g.w, mm.w, vv.w, lr, b1, b2, eps, bc1, bc2);
            *reinterpret_cast<float4 *>(m + i) = mm;
            *reinterpret_cast<float4 *>(v + i) = vv;
        } else {
            w.x = w.x - lr * g.x, w.y = w.y - lr * g.y, w.z = w.z - lr * g.z, w.w = w.w - lr * g.w;
        }
        uint2 o;
        if (out_bf16) {
            __nv_bfloat162 a0 = __floats2bfloat162_rn(w.x, w.y), a1 = __floats2bfloat162_rn(w.z, w.w);
            o.x = *reinterpret_cast<uint32_t *>(&a0);
            o.y = *reinterpret_cast<uint32_t *>(&a1);
        }
        for (int r = 0; r < nout; ++r) {
            *reinterpret_cast<float4 *>(out_f32[r] + i) = w;
            if (out_bf16) *reinterpret_cast<uint2 *>(out_bf16[r] + i) = o;
        }
    }
}

cudaError_t update_shard(const float *const *grads, int R, long lo, long hi, const float *w_in, float *const *out_f32,
                         __nv_bfloat16 *const *out_bf16, int nout, int opt, float *m, float *v, float lr, float b1, float b2,
                         float eps, int step, cudaStream_t s) {
    if ((lo & 3) || (hi & 3) || hi < lo) return cudaErrorInvalidValue;
    if (hi == lo) return cudaSuccess;
    const float bc1 = 1.f - powf(b1, (float)step), bc2 = 1.f - powf(b2, (float)step);
    const long n4 = (hi - lo) / 4;
    long blocks = (n4 + 255) / 256;
    if (blocks > 148L * 8) blocks = 148L * 8;
    if (opt == PD_ADAM)
        update_shard_kernel<true><<<(unsigned)blocks, 256, 0, s>>>(grads, R, lo, n4, w_in, out_f32, out_bf16, nout, m, v, lr, b1,
                                                                   b2, eps, bc1, bc2);
    else
        update_shard_kernel<false><<<(unsigned)blocks, 256, 0, s>>>(grads, R, lo, n4, w_in, out_f32, out_bf16, nout, m, v, lr,
                                                                    b1, b2, eps, bc1, bc2);
    ++tl_launches;
    return cudaGetLastError();
}

cudaError_t update_from_grad(float *master, __nv_bfloat16 *slot, const float *g, long n, int opt, float *m, float *v,
                             float lr, float b1, float b2, float eps, int step, cudaStream_t s) {
    if ((n & 3) || ((uintptr_t)master & 15) || ((uintptr_t)g & 15) || ((uintptr_t)slot & 7) ||
        (opt == PD_ADAM && (((uintptr_t)m & 15) || ((uintptr_t)v & 15))))
        return cudaErrorInvalidValue;
    const float bc1 = 1.f - powf(b1, (float)step), bc2 = 1.f - powf(b2, (float)step);
    const long n4 = n / 4;
    if (opt == PD_ADAM)
        update_vec4_kernel<true><<<grid_for(n4), 256, 0, s>>>(master, slot, g, n4, m, v, lr, b1, b2, eps, bc1, bc2);
    else
        update_vec4_kernel<false><<<grid_for(n4), 256, 0, s>>>(master, slot, g, n4, m, v, lr, b1, b2, eps, bc1, bc2);
    ++tl_launches;
    return cudaGetLastError();
}

namespace {
__global__ void regions_bf16_to_f32_kernel(const __nv_bfloat16 *__restrict__ src, float *__restrict__ dst,
                                           const long *__restrict__ off, const int *__restrict__ cnt) {
    const long o = off[blockIdx.y];
    const int n = cnt[blockIdx.y];
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
        dst[o + i] = __bfloat162float(src[o + i]);
}
}  // namespace

cudaError_t regions_bf16_to_f32(const __nv_bfloat16 *src, float *dst, const long *off, const int *cnt, int n,
                                cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    regions_bf16_to_f32_kernel<<<dim3(8, n), 256, 0, s>>>(src, dst, off, cnt);
    ++tl_launches;
    return cudaGetLastError();
}

cudaError_t f32_to_bf16(const float *in, __nv_bfloat16 *out, long n, cudaStream_t s) {
    f32_to_bf16_kernel<<<grid_for(n), 256, 0, s>>>(in, out, n);
    ++tl_launches;
    return cudaGetLastError();
}

cudaError_t bf16_to_f32(const __nv_bfloat16 *in, float *out, long n, cudaStream_t s) {
    bf16_to_f32_kernel<<<grid_for(n), 256, 0, s>>>(in, out, n);
    ++tl_launches;
    return cudaGetLastError();
}

// solo measurement mode: counter-hash values uniform in [-scale, scale) (content does not
// affect the kernels' speed, but all-zero operands would understate power draw)
__global__ void fill_uniform_kernel(void *p, long n, int bf16, float scale, uint32_t seed) {
    for (long i = (long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long)gridDim.x * blockDim.x) {
        uint32_t x = (uint32_t)i * 0x9E3779B9u ^ seed;
        x ^= x >> 16;
        x *= 0x7FEB352Du;
        x ^= x >> 15;
        x *= 0x846CA68Bu;
        x ^= x >> 16;
        const float v = scale * ((float)(x >> 8) * (2.f / 16777216.f) - 1.f);
        if (bf16) static_cast<__nv_bfloat16 *>(p)[i] = __float2bfloat16(v);
        else static_cast<float *>(p)[i] = v;
    }
}

cudaError_t fill_uniform(void *p, long n, int bf16, float scale, uint32_t seed, cudaStream_t s) {
    fill_uniform_kernel<<<grid_for(n), 256, 0, s>>>(p, n, bf16, scale, seed);
    ++tl_launches;
    return cudaGetLastError();
}

cudaError_t signal_flag(uint32_t *flag, uint32_t value, cudaStream_t s) {
    signal_kernel<<<1, 1, 0, s>>>(flag, value);
    ++tl_launches;
    return cudaGetLastError();
}

}  // namespace pd
