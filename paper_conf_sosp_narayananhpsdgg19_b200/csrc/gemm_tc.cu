// gemm_tc.cu -- bf16 x bf16 -> fp32 GEMM on the 5th-generation tensor cores (sm_100a).
//
//   C(m, n) = sum_k A(m, k) B(n, k), A/B each K-major or MN-major (so the forward
//   X W^T, the input gradient G W and the weight gradient G^T X of a linear layer all run
//   without transposes), with the layer epilogues fused:
//     EPI_STORE  out = act(acc + bias)            bf16   (forward; may be a peer pointer)
//     EPI_MASK   out = acc * (mask > 0)           bf16   (dX fused with ReLU derivative)
//     EPI_F32    out = acc                        fp32   (gradient for replica allreduce)
//     EPI_SGD    master -= lr acc; slot = bf16(master)   (dW fused with the update that
//     EPI_ADAM   Adam on master, m, v; slot = bf16(master) writes the next weight version)
//
// Structure (persistent, warp-specialised, one CTA per SM):
//   warp 0      TMA producer: cp.async.bulk.tensor 2-D tiles, 128B swizzle, into a
//               STAGES-deep shared-memory ring guarded by full/empty mbarriers;
//   warp 1      MMA issuer: one elected thread issues tcgen05.mma.cta_group::1.kind::f16
//               (M = 128, N = BN, K = 16) into a double-buffered TMEM accumulator and
//               tcgen05.commit's the smem slot / accumulator barriers;
//   warp 2      TMEM allocator (2 * BN columns);
//   warps 4..7  epilogue: tcgen05.ld 32 lanes x 32 columns -> registers -> fused op ->
//               16-byte global stores, overlapping the next tile's MMAs.
#include <cuda.h>
#include <cuda_bf16.h>

#include <cstdio>
#include <cstdlib>
#include <unordered_map>
#include <vector>
#include <algorithm>

#include "pd_internal.h"
#include "tc_ptx.h"

namespace pd {
namespace {

constexpr int BM = 128;
constexpr int BK = 64;  // 64 bf16 = 128 B = one swizzle row
constexpr int UMMA_K = 16;
constexpr int NUM_THREADS = 256;

enum { EPI_STORE_ = 0, EPI_MASK_ = 1, EPI_F32_ = 2 };  // (mirror of pd_internal.h's EPI_* for constexprs)
template <int BN, int EPI = 0>
struct Cfg {
    static constexpr int A_BYTES = BM * BK * 2;
    static constexpr int B_BYTES = BN * BK * 2;
    static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
    // epilogue staging per epilogue warp (TMA-store epilogue): two 32 x 32 output tiles (fp32
    // 4 KB or bf16 2 KB each, swizzled) + two bf16 mask tiles (EPI_MASK)
    static constexpr int OUT_TILE = EPI == EPI_F32_ ? 4096 : 2048;
    // (STORE / MASK also host the cluster split-K output slice: up to 4 x [128][32] bf16 = 32 KB)
    static constexpr int WARP_STG = EPI > EPI_F32_ ? 0 : (EPI == EPI_F32_ ? 2 * OUT_TILE : 8192);
    static constexpr int EPI_STG = 4 * WARP_STG;
    static constexpr int STAGES_MAX = (BN == 256) ? 4 : (BN == 128 ? 6 : 8);
    static constexpr int STAGES_FIT = (232448 - 1024 - 256 - EPI_STG) / STAGE_BYTES;
    static constexpr int STAGES = STAGES_FIT < STAGES_MAX ? STAGES_FIT : STAGES_MAX;
    static constexpr int TMEM_COLS = 2 * BN < 32 ? 32 : 2 * BN;
    static constexpr int SMEM = STAGES * STAGE_BYTES + EPI_STG + 1024 /*align*/ + 256 /*barriers*/;
};

struct EpiArgs {
    void *out;
    long ldo;
    long split_stride;  // elements between the fp32 partial outputs of K-splits (EPI_F32)
    int ksplit;         // K is cut into ksplit contiguous ranges; work unit = (tile, split)
    ConvGeom conv;      // implicit-GEMM 3x3 convolution geometry (conv.taps == 0: plain GEMM)
    int atomic_out;     // EPI_F32: accumulate with fp32 atomics (split-K / per-tap dW)
    unsigned long long *probe;  // tools only (PD_GEMM_PROBE): per-CTA %globaltimer phase stamps [grid][8]
    const unsigned *wait_cnt;   // Gemm::wait_cnt (splits run in reverse, each waits for its rows)
    int wait_T, wait_B;
    unsigned wait_per;
    const float *bias;
    int relu;
    const __nv_bfloat16 *mask;
    long ldm;
    float *master;
    __nv_bfloat16 *slot;
    float *adam_m, *adam_v;
    float lr, b1, b2, eps, bc1, bc2;
};

using namespace tcx;

// ---------------------------------------------------------------- epilogue
template <int EPI>
__device__ __forceinline__ void epilogue_chunk(const EpiArgs &e, float (&v)[32], int row, int col, int M, int N) {
    if (row >= M) return;
    const bool full = (col + 32 <= N);
    // conv output on the zero-padded grid: border pixels are written as 0 so buffers never
    // need clearing and the next layer's halo stays zero
    bool border = false;
    if (e.conv.Hp) {
        const int wp = row % e.conv.Wp, hp = (row / e.conv.Wp) % e.conv.Hp;
        border = hp == 0 || hp == e.conv.Hp - 1 || wp == 0 || wp == e.conv.Wp - 1;
    }
    if constexpr (EPI == EPI_STORE || EPI == EPI_MASK) {
        if constexpr (EPI == EPI_STORE) {
            if (e.bias) {
#pragma unroll
                for (int i = 0; i < 32; ++i) v[i] += (col + i < N) ? e.bias[col + i] : 0.f;
            }
            if (e.relu) {
#pragma unroll
                for (int i = 0; i < 32; ++i) v[i] = fmaxf(v[i], 0.f);
            }
            if (border) {
#pragma unroll
                for (int i = 0; i < 32; ++i) v[i] = 0.f;
            }
        } else {
            if (border) {
#pragma unroll
                for (int i = 0; i < 32; ++i) v[i] = 0.f;
            }
            const __nv_bfloat16 *mk = e.mask + (long)row * e.ldm + col;
            if (full) {
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    uint4 raw = *reinterpret_cast<const uint4 *>(mk + q * 8);
                    const __nv_bfloat16 *h = reinterpret_cast<const __nv_bfloat16 *>(&raw);
#pragma unroll
                    for (int i = 0; i < 8; ++i) v[q * 8 + i] = (__bfloat162float(h[i]) > 0.f) ? v[q * 8 + i] : 0.f;
                }
            } else {
                for (int i = 0; i < 32; ++i)
                    if (col + i < N) v[i] = (__bfloat162float(mk[i]) > 0.f) ? v[i] : 0.f;
            }
        }
        __nv_bfloat16 *o = static_cast<__nv_bfloat16 *>(e.out) + (long)row * e.ldo + col;
        if (full) {
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                uint4 w;
                w.x = pack_bf16(v[q * 8 + 0], v[q * 8 + 1]);
                w.y = pack_bf16(v[q * 8 + 2], v[q * 8 + 3]);
                w.z = pack_bf16(v[q * 8 + 4], v[q * 8 + 5]);
                w.w = pack_bf16(v[q * 8 + 6], v[q * 8 + 7]);
                *reinterpret_cast<uint4 *>(o + q * 8) = w;
            }
        } else {
            for (int i = 0; i < 32; ++i)
                if (col + i < N) o[i] = __float2bfloat16_rn(v[i]);
        }
    } else if constexpr (EPI == EPI_F32) {
        float *o = static_cast<float *>(e.out) + (long)row * e.ldo + col;
        if (e.atomic_out) {
            for (int i = 0; i < 32; ++i)
                if (col + i < N) atomicAdd(o + i, v[i]);
            return;
        }
        if (full) {
#pragma unroll
            for (int q = 0; q < 8; ++q)
                *reinterpret_cast<float4 *>(o + q * 4) = make_float4(v[q * 4], v[q * 4 + 1], v[q * 4 + 2], v[q * 4 + 3]);
        } else {
            for (int i = 0; i < 32; ++i)
                if (col + i < N) o[i] = v[i];
        }
    } else {  // EPI_SGD / EPI_ADAM: fused weight update writing the next version
        const long base = (long)row * e.ldo + col;
        float *ms = e.master + base;
        __nv_bfloat16 *sl = e.slot + base;
        if (full) {
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                float4 w = *reinterpret_cast<float4 *>(ms + q * 4);
                float g[4] = {v[q * 4], v[q * 4 + 1], v[q * 4 + 2], v[q * 4 + 3]};
                float wv[4] = {w.x, w.y, w.z, w.w};
                if constexpr (EPI == EPI_SGD) {
#pragma unroll
                    for (int i = 0; i < 4; ++i) wv[i] = wv[i] - e.lr * g[i];
                } else {
                    float4 m4 = *reinterpret_cast<float4 *>(e.adam_m + base + q * 4);
                    float4 v4 = *reinterpret_cast<float4 *>(e.adam_v + base + q * 4);
                    float mm[4] = {m4.x, m4.y, m4.z, m4.w}, vv[4] = {v4.x, v4.y, v4.z, v4.w};
#pragma unroll
                    for (int i = 0; i < 4; ++i) {
                        mm[i] = e.b1 * mm[i] + (1.f - e.b1) * g[i];
                        vv[i] = e.b2 * vv[i] + (1.f - e.b2) * g[i] * g[i];
                        wv[i] = wv[i] - e.lr * (mm[i] / e.bc1) / (sqrtf(vv[i] / e.bc2) + e.eps);
                    }
                    *reinterpret_cast<float4 *>(e.adam_m + base + q * 4) = make_float4(mm[0], mm[1], mm[2], mm[3]);
                    *reinterpret_cast<float4 *>(e.adam_v + base + q * 4) = make_float4(vv[0], vv[1], vv[2], vv[3]);
                }
                *reinterpret_cast<float4 *>(ms + q * 4) = make_float4(wv[0], wv[1], wv[2], wv[3]);
                uint2 p;
                p.x = pack_bf16(wv[0], wv[1]);
                p.y = pack_bf16(wv[2], wv[3]);
                *reinterpret_cast<uint2 *>(sl + q * 4) = p;
            }
        } else {
            for (int i = 0; i < 32; ++i) {
                if (col + i >= N) continue;
                float w = ms[i];
                if constexpr (EPI == EPI_SGD) {
                    w = w - e.lr * v[i];
                } else {
                    float mm = e.adam_m[base + i], vv = e.adam_v[base + i];
                    mm = e.b1 * mm + (1.f - e.b1) * v[i];
                    vv = e.b2 * vv + (1.f - e.b2) * v[i] * v[i];
                    w = w - e.lr * (mm / e.bc1) / (sqrtf(vv / e.bc2) + e.eps);
                    e.adam_m[base + i] = mm;
                    e.adam_v[base + i] = vv;
                }
                ms[i] = w;
                sl[i] = __float2bfloat16_rn(w);
            }
        }
    }
}


// TMA-store epilogue (STORE / MASK / F32).  Each epilogue warp owns 32 accumulator rows; a
// 32 x 32 chunk (lane = row) gets its elementwise op in registers, is written to a swizzled
// shared tile (16-byte stores, conflict-free) and leaves with ONE bulk tensor store (or an
// L2-side fp32 reduce-add for split-K / per-tap partial sums), double-buffered so the next
// chunk's TMEM load overlaps the store.  Plain st.global from 4 warps per SM sustained only
// ~13 B/clk (latency bound); the TMA engine keeps many stores in flight.
__device__ __forceinline__ uint32_t stg_off_f32(int r, int j) { return r * 128 + ((j ^ (r & 7)) << 4); }
__device__ __forceinline__ uint32_t stg_off_bf16(int r, int j) { return r * 64 + ((j ^ ((r >> 1) & 3)) << 4); }

template <int EPI>
__device__ __forceinline__ void epi_math(const EpiArgs &e, float (&v)[32], int row, int col, int N,
                                         const uint8_t *mask_tile, int lane) {
    bool border = false;
    if (e.conv.Hp) {
        const int wp = row % e.conv.Wp, hp = (row / e.conv.Wp) % e.conv.Hp;
        border = hp == 0 || hp == e.conv.Hp - 1 || wp == 0 || wp == e.conv.Wp - 1;
    }
    if constexpr (EPI == EPI_STORE) {
        if (e.bias) {
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] += (col + i < N) ? __ldg(e.bias + col + i) : 0.f;
        }
        if (e.relu) {
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] = fmaxf(v[i], 0.f);
        }
    } else if constexpr (EPI == EPI_MASK) {
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const uint4 raw = *reinterpret_cast<const uint4 *>(mask_tile + stg_off_bf16(lane, j));
            const __nv_bfloat16 *h = reinterpret_cast<const __nv_bfloat16 *>(&raw);
#pragma unroll
            for (int i = 0; i < 8; ++i) v[j * 8 + i] = (__bfloat162float(h[i]) > 0.f) ? v[j * 8 + i] : 0.f;
        }
    }
    if (EPI != EPI_F32 && border) {
#pragma unroll
        for (int i = 0; i < 32; ++i) v[i] = 0.f;
    }
}

template <int EPI>
__device__ __forceinline__ void epi_stage(uint8_t *tile, const float (&v)[32], int lane) {
    if constexpr (EPI == EPI_F32) {
#pragma unroll
        for (int j = 0; j < 8; ++j)
            *reinterpret_cast<float4 *>(tile + stg_off_f32(lane, j)) =
                make_float4(v[4 * j], v[4 * j + 1], v[4 * j + 2], v[4 * j + 3]);
    } else {
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            uint4 w;
            w.x = pack_bf16(v[8 * j + 0], v[8 * j + 1]);
            w.y = pack_bf16(v[8 * j + 2], v[8 * j + 3]);
            w.z = pack_bf16(v[8 * j + 4], v[8 * j + 5]);
            w.w = pack_bf16(v[8 * j + 6], v[8 * j + 7]);
            *reinterpret_cast<uint4 *>(tile + stg_off_bf16(lane, j)) = w;
        }
    }
}

__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
#define PROBE(i)                                                   \
    do {                                                           \
        if (e.probe) e.probe[blockIdx.x * 16 + (i)] = gtimer();    \
    } while (0)

// ---------------------------------------------------------------- the kernel
// CG = 1: one CTA per 128 x BN tile.  CG = 2: a CTA pair (cluster of 2 on one TPC) per
// 256 x BN tile with tcgen05.mma.cta_group::2 -- each CTA stages its 128 rows of A and half
// (BN/2) of B, the leader issues the M = 256 MMAs reading both CTAs' shared memory, and
// each CTA's TMEM receives its 128 accumulator rows.  Per SM that halves the B bytes per
// FLOP, the lever that matters when the L2->SM fill (~80 GB/s per SM) is the limit.
template <int BN, int AMAJ, int BMAJ, int EPI, int CG>
__global__ void __launch_bounds__(NUM_THREADS, 1)
    tc_gemm_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                   const __grid_constant__ CUtensorMap tmO, const __grid_constant__ CUtensorMap tmK, EpiArgs e,
                   int M, int N, int K) {
    using C = Cfg<BN / CG, EPI>;  // shared-memory ring holds this CTA's A rows and B columns
    constexpr int BNC = BN / CG;
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    uint8_t *epi_stg = smem + C::STAGES * C::STAGE_BYTES;  // 1024-aligned (ring stages are)
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem + C::STAGES * C::STAGE_BYTES + C::EPI_STG);
    uint64_t *full = bars, *empty = bars + C::STAGES, *tfull = bars + 2 * C::STAGES, *tempty = tfull + 2;
    uint64_t *mbar = tempty + 2;  // [4 warps][2] mask-tile barriers (EPI_MASK)
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(mbar + 8);

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) PROBE(0);
    uint32_t crank = 0;  // rank in the CTA pair's cluster
    if (CG == 2) asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(crank));
    const uint32_t rank = CG == 2 ? (crank & 1u) : 0u;                  // rank in the CTA pair
    const uint16_t pmask = (uint16_t)(3u << (crank & ~1u));              // the pair's CTAs
    const int pair = blockIdx.x / CG, npairs = gridDim.x / CG;
    const int m_blocks = (M + BM * CG - 1) / (BM * CG), n_blocks = (N + BN - 1) / BN;
    const int tiles = m_blocks * n_blocks;
    const int kblocks = (K + BK - 1) / BK;
    const int units = tiles * e.ksplit;
    const int kper = (kblocks + e.ksplit - 1) / e.ksplit;
    // persistent loop over units (tile, split)
    const int u0 = pair, ustep = npairs;
    constexpr uint32_t TMEM_COLS = 2 * BN < 32 ? 32 : 2 * BN;

    if (warp == 0 && lane == 0) {
        asm volatile("prefetch.tensormap [%0];" ::"l"(&tmA) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(&tmB) : "memory");
        for (int s = 0; s < C::STAGES; ++s) {
            mbar_init(smem_u32(&full[s]), 1);
            mbar_init(smem_u32(&empty[s]), 1);
        }
        for (int a = 0; a < 2; ++a) {
            mbar_init(smem_u32(&tfull[a]), 1);
            mbar_init(smem_u32(&tempty[a]), 4 * CG);  // one arrival per epilogue warp of the pair
        }
        for (int a = 0; a < 8; ++a) mbar_init(smem_u32(&mbar[a]), 1);
        if (EPI == EPI_STORE || EPI == EPI_MASK || EPI == EPI_F32) {
            asm volatile("prefetch.tensormap [%0];" ::"l"(&tmO) : "memory");
            if (EPI == EPI_MASK) asm volatile("prefetch.tensormap [%0];" ::"l"(&tmK) : "memory");
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 2) {
        if (CG == 1) {
            asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                             smem_u32(tmem_slot)),
                         "r"(TMEM_COLS));
            asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
        } else {
            asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                             smem_u32(tmem_slot)),
                         "r"(TMEM_COLS));
            asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
        }
    }
    if (e.conv.c8 == 1) {
        // packed-tap forward: A slot 9 (K 72..79) is never loaded; it meets zero weights,
        // so it only has to be finite -- zero it once
        for (int s = 0; s < C::STAGES; ++s)
            for (int i = threadIdx.x; i < 2048 / 16; i += NUM_THREADS)
                reinterpret_cast<uint4 *>(smem + s * C::STAGE_BYTES + 9 * 2048)[i] = make_uint4(0, 0, 0, 0);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    }
    tc_fence_before();
    if (CG == 2) {
        asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory");
        asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory");
    } else {
        __syncthreads();
    }
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;
    if (threadIdx.x == 0) PROBE(1);

    if (warp == 0) {
        // ===== TMA producer =====
        if (lane == 0) {
            int stage = 0;
            uint32_t phase = 0;
            for (int unit = u0; unit < units; unit += ustep) {
                const int tile = unit % tiles, split = e.wait_cnt ? e.ksplit - 1 - unit / tiles : unit / tiles;
                const int m0 = (tile % m_blocks) * (BM * CG) + (int)rank * BM;
                const int n0 = (tile / m_blocks) * BN + (int)rank * BNC;
                const int kb0 = split * kper, kb1 = min(kblocks, kb0 + kper);
                if (e.wait_cnt && kb1 > kb0) {
                    // the rows of this split were produced by a kernel still running (the LSTM
                    // backward wave): wait for the producer's step counter, then the async proxy
                    const unsigned target = (unsigned)(e.wait_T - (kb0 * BK) / e.wait_B) * e.wait_per;
                    unsigned v;
                    const unsigned long long t0 = gtimer();
                    do {
                        asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(e.wait_cnt) : "memory");
                        if (gtimer() - t0 > 4000000000ull) __trap();  // (the producer kernel died)
                    } while (v < target);
                    asm volatile("fence.proxy.async.global;" ::: "memory");
                }
                // coordinates of K-block kb for this CTA (plain GEMM, implicit conv, shifted dW)
                auto coords = [&](int kb, int &ka, int &ma, int &kbk, int &nb) {
                    const int k0 = kb * BK;
                    ka = k0; ma = m0; kbk = k0; nb = n0;
                    if (e.conv.taps) {
                        const int tap = kb / e.conv.kpt, cblk = (kb % e.conv.kpt) * BK;
                        ka = cblk;
                        ma = m0 + e.conv.a_shift[tap];
                        kbk = cblk + tap * e.conv.b_koff;
                        nb = n0 + tap * e.conv.b_noff;
                    }
                    kbk += e.conv.b_kshift;
                };
                for (int kb = kb0; kb < kb1; ++kb) {
                    mbar_wait(smem_u32(&empty[stage]), phase ^ 1);
                    if (kb == kb0 && unit == u0) PROBE(2);
                    // CG = 2: both CTAs' bytes land on the LEADER's full barrier (peer bit cleared)
                    const uint32_t fb = smem_u32(&full[stage]) & (CG == 2 ? 0xFEFFFFFFu : 0xFFFFFFFFu);
                    const uint32_t sa = smem_u32(smem + stage * C::STAGE_BYTES);
                    const uint32_t sb = sa + C::A_BYTES;
                    if (CG == 1 && e.conv.c8 == 1) {
                        // packed-tap forward: A slot t = X rows shifted by tap t (2 KB each),
                        // B slot j = W[:, 8j .. 8j+7] (slot 9 past K = 72: zero fill)
                        mbar_expect_tx(fb, 9 * 2048 + 10 * BN / 2 * 16);
                        for (int t = 0; t < 9; ++t) tma_load_2d(sa + t * 2048, &tmA, fb, 0, m0 + e.conv.a_shift[t]);
                        for (int j = 0; j < 10; ++j) tma_load_2d(sa + 20480 + j * (BN / 2) * 16, &tmB, fb, 8 * j, n0);
                        if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
                        continue;
                    }
                    if (CG == 1 && e.conv.c8 == 2) {
                        // packed-tap dW: B slot t = 64 pixels of X shifted by tap t, 8 channels
                        const int k0 = kb * BK;
                        mbar_expect_tx(fb, C::A_BYTES + 9 * 1024);
#pragma unroll
                        for (int j = 0; j < BM / 64; ++j) tma_load_2d(sa + j * BK * 128, &tmA, fb, m0 + 64 * j, k0);
                        for (int t = 0; t < 9; ++t) tma_load_2d(sb + t * 1024, &tmB, fb, 0, k0 + e.conv.a_shift[t]);
                        if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
                        continue;
                    }
                    if (rank == 0) mbar_expect_tx(fb, CG * C::STAGE_BYTES);
                    // implicit-GEMM convolution: K-block kb = (tap, 64-channel block); the A rows
                    // (padded-grid pixels) shift by the tap's offset, B moves to the tap's slice
                    int ka, ma, kbk, nb;
                    coords(kb, ka, ma, kbk, nb);
                    if (AMAJ == KMAJ) {
                        tma_load_2d_cg<CG>(sa, &tmA, fb, ka, ma);  // box {64 K, 128 M}
                    } else {
#pragma unroll
                        for (int j = 0; j < BM / 64; ++j)
                            tma_load_2d_cg<CG>(sa + j * BK * 128, &tmA, fb, ma + 64 * j, ka);
                    }
                    if (BMAJ == KMAJ) {
                        tma_load_2d_cg<CG>(sb, &tmB, fb, kbk, nb);  // box {64 K, BN/CG N}
                    } else if (e.conv.b_tapchunk) {
                        // implicit im2col on B: column chunk (tap, 64 channels) = X rows shifted by the tap
                        const int Cp = e.conv.b_tapchunk;
#pragma unroll
                        for (int j = 0; j < BNC / 64; ++j) {
                            const int col = nb + 64 * j, tap = col / Cp;
                            if (tap < 9) tma_load_2d_cg<CG>(sb + j * BK * 128, &tmB, fb, col % Cp, kbk + e.conv.a_shift[tap]);
                            else tma_load_2d_cg<CG>(sb + j * BK * 128, &tmB, fb, Cp, kbk);  // past N: zero fill
                        }
                    } else {
#pragma unroll
                        for (int j = 0; j < BNC / 64; ++j)
                            tma_load_2d_cg<CG>(sb + j * BK * 128, &tmB, fb, nb + 64 * j, kbk);
                    }
                    if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
                }
            }
        }
    } else if (warp == 1) {
        // ===== MMA issuer (the pair's leader only) =====
        if (lane == 0 && rank == 0) {
            constexpr uint32_t idesc = make_idesc(BM * CG, BN, AMAJ, BMAJ);
            int stage = 0;
            uint32_t phase = 0;
            int acc = 0;
            uint32_t acc_phase = 0;
            for (int unit = u0; unit < units; unit += ustep) {
                const int split = e.wait_cnt ? e.ksplit - 1 - unit / tiles : unit / tiles;
                const int kb0 = split * kper, kb1 = min(kblocks, kb0 + kper);
                mbar_wait(smem_u32(&tempty[acc]), acc_phase ^ 1);
                tc_fence_after();
                const uint32_t d = tmem_base + acc * BN;
                for (int kb = kb0; kb < kb1; ++kb) {
                    mbar_wait(smem_u32(&full[stage]), phase);
                    tc_fence_after();
                    if (kb == kb0 && unit == u0) PROBE(3);
                    if (kb == kb0 + 1 && unit == u0) PROBE(7);
                    const uint32_t sa = smem_u32(smem + stage * C::STAGE_BYTES);
                    const uint32_t sb = sa + C::A_BYTES;
                    if (CG == 1 && e.conv.c8 == 1) {
                        // K = 80 in 5 steps; each step's two 8-wide K chunks are 2 slots apart
                        constexpr uint32_t id64 = make_idesc(BM, BN / 2, KMAJ, KMAJ);
                        for (int k = 0; k < 5; ++k) {
                            const uint64_t ad = smem_desc_ns(sa + k * 4096, 2048, 128);
                            const uint64_t bd = smem_desc_ns(sa + 20480 + k * 2 * (BN / 2) * 16, (BN / 2) * 16, 128);
                            tc_mma(d, ad, bd, id64, k > 0 ? 1u : 0u);
                        }
                        tc_commit(smem_u32(&empty[stage]));
                        if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
                        continue;
                    }
                    if (CG == 1 && e.conv.c8 == 2) {
                        // N = 80 (72 used): B is MN-major unswizzled, 8-pixel K groups 128 B apart,
                        // 8-channel N groups (taps) 1 KB apart
                        constexpr uint32_t id80 = make_idesc(BM, 80, MNMAJ, MNMAJ);
                        for (int k = 0; k < BK / UMMA_K; ++k) {
                            const uint64_t ad = smem_desc(sa + k * 2048, BK * 128, 1024);
                            const uint64_t bd = smem_desc_ns(sb + k * 256, 128, 1024);
                            tc_mma(d, ad, bd, id80, (kb > kb0 || k > 0) ? 1u : 0u);
                        }
                        tc_commit(smem_u32(&empty[stage]));
                        if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
                        continue;
                    }
#pragma unroll
                    for (int k = 0; k < BK / UMMA_K; ++k) {
                        const uint64_t ad = AMAJ == KMAJ ? smem_desc(sa + k * 32, 16, 1024)
                                                         : smem_desc(sa + k * 2048, BK * 128, 1024);
                        const uint64_t bd = BMAJ == KMAJ ? smem_desc(sb + k * 32, 16, 1024)
                                                         : smem_desc(sb + k * 2048, BK * 128, 1024);
                        tc_mma_cg<CG>(d, ad, bd, idesc, (kb > kb0 || k > 0) ? 1u : 0u);
                    }
                    tc_commit_cg<CG>(smem_u32(&empty[stage]), pmask);  // frees the slot (both CTAs) when done
                    if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
                }
                PROBE(4);
                tc_commit_cg<CG>(smem_u32(&tfull[acc]), pmask);  // accumulator ready for both epilogues
                if (++acc == 2) { acc = 0; acc_phase ^= 1; }
            }
        }
    } else if (warp >= 4) {
        // ===== epilogue =====
        const int q = warp & 3;  // TMEM lane quarter this warp may access
        int acc = 0;
        uint32_t acc_phase = 0;
        uint32_t ocnt = 0, mcnt = 0, mph = 0;  // staging-buffer / mask-buffer counters and phases
        for (int unit = u0; unit < units; unit += ustep) {
            const int tile = unit % tiles, split = e.wait_cnt ? e.ksplit - 1 - unit / tiles : unit / tiles;
            const int m0 = (tile % m_blocks) * (BM * CG) + (int)rank * BM, n0 = (tile / m_blocks) * BN;
            mbar_wait(smem_u32(&tfull[acc]), acc_phase);
            tc_fence_after();
            if (warp == 4 && lane == 0) PROBE(5);
            const int row = m0 + q * 32 + lane;
            EpiArgs es = e;
            if (EPI == EPI_F32) es.out = static_cast<float *>(e.out) + (long)split * e.split_stride;
            const bool empty_range = split * kper >= kblocks;  // (host avoids it; be safe)
            if (EPI == EPI_STORE || EPI == EPI_MASK || EPI == EPI_F32) {
                // ---- TMA-store epilogue: rows m0+32q.., one 32 x 32 chunk at a time
                uint8_t *wst = epi_stg + q * C::WARP_STG;
                const int r0 = m0 + q * 32;
                const int nch = min(BN / 32, (N - n0 + 31) / 32);
                if (EPI == EPI_MASK && lane == 0 && nch > 0) {
                    uint8_t *mt = wst + 2 * C::OUT_TILE + (mcnt & 1) * 2048;
                    mbar_expect_tx(smem_u32(&mbar[q * 2 + (mcnt & 1)]), 2048);
                    tma_load_2d(smem_u32(mt), &tmK, smem_u32(&mbar[q * 2 + (mcnt & 1)]), n0, r0);
                }
#pragma unroll 1
                for (int c = 0; c < nch; ++c) {
                    if (EPI == EPI_MASK && lane == 0 && c + 1 < nch) {
                        // prefetch the next chunk's mask tile into the other buffer
                        const uint32_t nb = (mcnt + 1) & 1;
                        mbar_expect_tx(smem_u32(&mbar[q * 2 + nb]), 2048);
                        tma_load_2d(smem_u32(wst + 2 * C::OUT_TILE + nb * 2048), &tmK, smem_u32(&mbar[q * 2 + nb]),
                                    n0 + (c + 1) * 32, r0);
                    }
                    float v[32];
                    tmem_ld32(tmem_base + ((uint32_t)(q * 32) << 16) + acc * BN + c * 32, v);
                    if (warp == 4 && lane == 0 && c == 0) PROBE(8);
                    if (empty_range && e.atomic_out) continue;
                    if (empty_range) {
#pragma unroll
                        for (int i = 0; i < 32; ++i) v[i] = 0.f;
                    }
                    const uint8_t *mt = nullptr;
                    if constexpr (EPI == EPI_MASK) {
                        const uint32_t b = mcnt & 1;
                        mbar_wait(smem_u32(&mbar[q * 2 + b]), (mph >> b) & 1);
                        mph ^= 1u << b;
                        mt = wst + 2 * C::OUT_TILE + b * 2048;
                    }
                    epi_math<EPI>(es, v, row, n0 + c * 32, N, mt, lane);
                    if constexpr (EPI == EPI_MASK) {
                        __syncwarp();  // every lane has read this mask buffer before it is refilled
                        ++mcnt;
                    }
                    // the store issued two chunks ago has finished reading this staging buffer
                    if (lane == 0) bulk_wait_read1();
                    __syncwarp();
                    uint8_t *ot = wst + (ocnt & 1) * C::OUT_TILE;
                    epi_stage<EPI>(ot, v, lane);
                    fence_proxy_async();
                    __syncwarp();
                    if (lane == 0) {
                        if (EPI == EPI_F32 && e.atomic_out) tma_reduce_add_2d(&tmO, smem_u32(ot), n0 + c * 32, r0);
                        else if (EPI == EPI_F32 && e.split_stride) tma_store_3d(&tmO, smem_u32(ot), n0 + c * 32, r0, split);
                        else tma_store_2d(&tmO, smem_u32(ot), n0 + c * 32, r0);
                        bulk_commit();
                    }
                    ++ocnt;
                    if (warp == 4 && lane == 0 && c < 2) PROBE(9 + c);
                }
            } else {
#pragma unroll 1
            for (int c = 0; c < BN / 32; ++c) {
                float v[32];
                tmem_ld32(tmem_base + ((uint32_t)(q * 32) << 16) + acc * BN + c * 32, v);
                if (empty_range) {
                    if (e.atomic_out) continue;
#pragma unroll
                    for (int i = 0; i < 32; ++i) v[i] = 0.f;
                }
                if (n0 + c * 32 < N) epilogue_chunk<EPI>(es, v, row, n0 + c * 32, M, N);
            }
            }
            if (warp == 4 && lane == 0) PROBE(11);
            tc_fence_before();
            __syncwarp();
            if (lane == 0) {
                if (CG == 1) mbar_arrive(smem_u32(&tempty[acc]));
                else mbar_arrive_cluster(smem_u32(&tempty[acc]) & 0xFEFFFFFFu);  // the leader's barrier
            }
            if (++acc == 2) { acc = 0; acc_phase ^= 1; }
        }
        if (EPI == EPI_STORE || EPI == EPI_MASK || EPI == EPI_F32) {
            if (lane == 0) bulk_wait0();  // every bulk store complete before the CTA retires
        }
        if (warp == 4 && lane == 0) PROBE(6);
    }
    tc_fence_before();
    if (CG == 2) {
        asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory");
        asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory");
    } else {
        __syncthreads();
    }
    if (warp == 2) {
        tc_fence_after();
        if (CG == 1)
            asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(TMEM_COLS));
        else
            asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(TMEM_COLS));
    }
}

// ---------------------------------------------------------------- small-M GEMM: cluster split-K
// The forward X W^T and input-gradient G W of a minibatch (M = B = 256 rows) have only
// 2 x N/256 output tiles; a K-split restores the parallelism.  Here the S K-splits of one
// 128 x 256 output tile are the S CTAs of one thread-block cluster, and their fp32 partial
// tiles never leave the chip: after the main loops every CTA owns 256/S output columns,
// sends its partials of the other columns to their owners' shared memory (one bulk DSMEM
// copy per peer, completing on the owner's mbarrier), sums the S partials of its own columns
// in split order (deterministic), applies the layer epilogue (bias + ReLU, or the ReLU mask of
// the layer below) and stores bf16 with TMA.  One launch, no fp32 workspace in HBM, no
// reduction kernel (the unclustered split-K path wrote S fp32 partial sets and re-read them).
//   smem: the operand ring (4 x 48 KB); after the main loop the ring holds the outbox
//   ((S-1) slices) and the receive slots ((S-1) slices), a slice = 128 rows x 256/S columns
//   fp32, 16-byte chunks XOR-swizzled by row (conflict-free: a warp's lanes are 32 rows).
template <int AMAJ, int BMAJ, int EPI, int S>
__global__ void __launch_bounds__(NUM_THREADS, 1)
    tc_gemm_csplit_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                          const __grid_constant__ CUtensorMap tmO, const __grid_constant__ CUtensorMap tmK, EpiArgs e,
                          int M, int N, int K) {
    constexpr int BN = 256;
    using C = Cfg<BN, EPI>;
    constexpr int W = BN / S;                 // output columns each CTA owns
    constexpr uint32_t SLICE = 128u * W * 4;  // one partial slice (bytes)
    static_assert(2 * (S - 1) * SLICE <= (uint32_t)C::STAGES * C::STAGE_BYTES, "exchange does not fit the ring");
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    uint8_t *epi_stg = smem + C::STAGES * C::STAGE_BYTES;
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem + C::STAGES * C::STAGE_BYTES + C::EPI_STG);
    uint64_t *full = bars, *empty = bars + C::STAGES, *tfull = bars + 2 * C::STAGES, *rbar = tfull + 1;
    uint64_t *mbar = rbar + 1;  // [4 warps][2] mask-tile barriers (EPI_MASK)
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(mbar + 8);
    uint8_t *outbox = smem;                          // (S-1) slices, by peer order
    uint8_t *recv = smem + (S - 1) * SLICE;          // (S-1) slices, by sender order

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) PROBE(0);
    uint32_t r;  // split index = rank in the cluster
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    const int tile = blockIdx.x / S;
    const int m_blocks = (M + BM - 1) / BM;
    const int m0 = (tile % m_blocks) * BM, n0 = (tile / m_blocks) * BN;
    const int kblocks = (K + BK - 1) / BK;
    const int kper = (kblocks + S - 1) / S;
    const int kb0 = (int)r * kper, kb1 = min(kblocks, kb0 + kper);

    if (warp == 0 && lane == 0) {
        asm volatile("prefetch.tensormap [%0];" ::"l"(&tmA) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(&tmB) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(&tmO) : "memory");
        if (EPI == EPI_MASK) asm volatile("prefetch.tensormap [%0];" ::"l"(&tmK) : "memory");
        for (int s = 0; s < C::STAGES; ++s) {
            mbar_init(smem_u32(&full[s]), 1);
            mbar_init(smem_u32(&empty[s]), 1);
        }
        mbar_init(smem_u32(tfull), 1);
        mbar_init(smem_u32(rbar), 1);
        for (int a = 0; a < 8; ++a) mbar_init(smem_u32(&mbar[a]), 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 2) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                     "r"(BN));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    tc_fence_before();
    cluster_sync_all();  // every CTA's barriers exist before any peer copy can target them
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;
    if (threadIdx.x == 0) PROBE(1);
    // the receive barrier's phase 0 completes when all (S-1) peer slices have landed
    if (warp == 0 && lane == 0) mbar_expect_tx(smem_u32(rbar), (S - 1) * SLICE);

    if (warp == 0) {
        if (lane == 0) {  // ===== TMA producer
            int stage = 0;
            uint32_t phase = 0;
            for (int kb = kb0; kb < kb1; ++kb) {
                mbar_wait(smem_u32(&empty[stage]), phase ^ 1);
                const uint32_t fb = smem_u32(&full[stage]);
                const uint32_t sa = smem_u32(smem + stage * C::STAGE_BYTES), sb = sa + C::A_BYTES;
                mbar_expect_tx(fb, C::STAGE_BYTES);
                const int k0 = kb * BK;
                if (AMAJ == KMAJ) {
                    tma_load_2d(sa, &tmA, fb, k0, m0);
                } else {
#pragma unroll
                    for (int j = 0; j < BM / 64; ++j) tma_load_2d(sa + j * BK * 128, &tmA, fb, m0 + 64 * j, k0);
                }
                if (BMAJ == KMAJ) {
                    tma_load_2d(sb, &tmB, fb, k0, n0);
                } else {
#pragma unroll
                    for (int j = 0; j < BN / 64; ++j) tma_load_2d(sb + j * BK * 128, &tmB, fb, n0 + 64 * j, k0);
                }
                if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
            }
        }
    } else if (warp == 1) {
        if (lane == 0) {  // ===== MMA issuer
            constexpr uint32_t idesc = make_idesc(BM, BN, AMAJ, BMAJ);
            int stage = 0;
            uint32_t phase = 0;
            for (int kb = kb0; kb < kb1; ++kb) {
                mbar_wait(smem_u32(&full[stage]), phase);
                tc_fence_after();
                if (kb == kb0) PROBE(3);
                const uint32_t sa = smem_u32(smem + stage * C::STAGE_BYTES), sb = sa + C::A_BYTES;
#pragma unroll
                for (int k = 0; k < BK / UMMA_K; ++k) {
                    const uint64_t ad = AMAJ == KMAJ ? smem_desc(sa + k * 32, 16, 1024) : smem_desc(sa + k * 2048, BK * 128, 1024);
                    const uint64_t bd = BMAJ == KMAJ ? smem_desc(sb + k * 32, 16, 1024) : smem_desc(sb + k * 2048, BK * 128, 1024);
                    tc_mma(tmem_base, ad, bd, idesc, (kb > kb0 || k > 0) ? 1u : 0u);
                }
                tc_commit(smem_u32(&empty[stage]));
                if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
            }
            PROBE(4);
            tc_commit(smem_u32(tfull));  // (kb1 > kb0: the host never makes an empty split)
        }
    } else if (warp >= 4) {
        mbar_wait(smem_u32(tfull), 0);
        tc_fence_after();
        if (warp == 4 && lane == 0) PROBE(5);
    }
    // every CTA's MMAs are complete: all operand rings are free for the exchange
    tc_fence_before();
    cluster_sync_all();
    tc_fence_after();

    if (warp >= 4) {
        if (warp == 4 && lane == 0) PROBE(7);  // (after the cluster barrier)
        const int q = warp & 3;
        const int row = q * 32 + lane;  // accumulator row (TMEM lane) of this thread
        const uint32_t tl = tmem_base + ((uint32_t)(q * 32) << 16);
        auto slice_off = [&](int col) {  // byte offset of (row, col..col+3) in a slice
            const int jj = col >> 2;
            return (uint32_t)row * (W * 4) + (uint32_t)((jj ^ (row & 15)) << 4);
        };
        // ---- partials of the peers' columns -> outbox slice (peer order) -> one bulk copy each
#pragma unroll 1
        for (int p = 0; p < S; ++p) {
            if (p == (int)r) continue;
            uint8_t *slc = outbox + (p < (int)r ? p : p - 1) * SLICE;
#pragma unroll 1
            for (int c = 0; c < W / 32; ++c) {
                float v[32];
                tmem_ld32(tl + p * W + c * 32, v);
#pragma unroll
                for (int i = 0; i < 8; ++i)
                    st_shared_v4(smem_u32(slc) + slice_off(c * 32 + 4 * i), v[4 * i], v[4 * i + 1], v[4 * i + 2],
                                 v[4 * i + 3]);
            }
        }
        fence_proxy_async();
        asm volatile("bar.sync 1, 128;" ::: "memory");  // the 128 epilogue threads have written the outbox
        if (warp == 4 && lane == 0) {
            for (int p = 0; p < S; ++p) {
                if (p == (int)r) continue;
                const uint32_t src = smem_u32(outbox + (p < (int)r ? p : p - 1) * SLICE);
                const uint32_t dst = mapa_cluster(smem_u32(recv + ((int)r < p ? (int)r : (int)r - 1) * SLICE), p);
                const uint32_t pb = mapa_cluster(smem_u32(rbar), p);
                asm volatile(
                    "cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                        dst),
                    "r"(src), "r"(SLICE), "r"(pb)
                    : "memory");
            }
        }
        // ---- own columns: sum the S partials in split order, epilogue, bf16 TMA store
        if (warp == 4 && lane == 0) PROBE(8);
        mbar_wait(smem_u32(rbar), 0);
        if (warp == 4 && lane == 0) PROBE(9);
        uint8_t *wst = epi_stg + q * C::WARP_STG;
        const int r0 = m0 + q * 32;
        const int nc = n0 + (int)r * W;  // first owned column
        uint32_t ocnt = 0;
#pragma unroll 1
        for (int c = 0; c < W / 32; ++c) {
            const int col = nc + c * 32;
            if (col >= N) break;
            if (EPI == EPI_MASK && lane == 0) {
                mbar_expect_tx(smem_u32(&mbar[q * 2 + (c & 1)]), 2048);
                tma_load_2d(smem_u32(wst + 2 * C::OUT_TILE + (c & 1) * 2048), &tmK, smem_u32(&mbar[q * 2 + (c & 1)]),
                            col, r0);
            }
            float own[32], v[32];
            tmem_ld32(tl + (int)r * W + c * 32, own);
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] = 0.f;
#pragma unroll 1
            for (int sp = 0; sp < S; ++sp) {
                if (sp == (int)r) {
#pragma unroll
                    for (int i = 0; i < 32; ++i) v[i] += own[i];
                } else {
                    const uint8_t *slc = recv + (sp < (int)r ? sp : sp - 1) * SLICE;
#pragma unroll
                    for (int i = 0; i < 8; ++i) {
                        const float4 x = *reinterpret_cast<const float4 *>(slc + slice_off(c * 32 + 4 * i));
                        v[4 * i] += x.x, v[4 * i + 1] += x.y, v[4 * i + 2] += x.z, v[4 * i + 3] += x.w;
                    }
                }
            }
            const uint8_t *mt = nullptr;
            if constexpr (EPI == EPI_MASK) {
                mbar_wait(smem_u32(&mbar[q * 2 + (c & 1)]), (c >> 1) & 1);
                mt = wst + 2 * C::OUT_TILE + (c & 1) * 2048;
            }
            epi_math<EPI>(e, v, r0 + lane, col, N, mt, lane);
            if (lane == 0) bulk_wait_read1();  // the store two chunks ago has read this buffer
            __syncwarp();
            uint8_t *ot = wst + (ocnt & 1) * C::OUT_TILE;
            epi_stage<EPI>(ot, v, lane);
            fence_proxy_async();
            __syncwarp();
            if (lane == 0) {
                tma_store_2d(&tmO, smem_u32(ot), col, r0);
                bulk_commit();
            }
            ++ocnt;
        }
        if (lane == 0) bulk_wait0();
        if (warp == 4 && lane == 0) PROBE(11);
    }
    // no CTA leaves while a peer may still copy into / out of its shared memory
    tc_fence_before();
    cluster_sync_all();
    if (threadIdx.x == 0) PROBE(6);
    if (warp == 2) {
        tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(BN));
    }
}

// Pair variant (the default for M <= 256-row tiles): a cluster of 4 = two CTA pairs.  Each
// pair runs cta_group::2 MMAs on a 256 x 128 tile (each CTA stages its 128 rows of A and 64
// of the 128 B columns: 24 KB per K-block instead of 48 KB), the two pairs take the two K
// halves, and CTA (pair rank p, split s) owns the 64 columns 64s..64s+63 of its 128 rows: it
// sends the other 64 columns' partials (32 KB) to the CTA of the other split with the same
// rows.  Per CTA: 768 KB of operands over half the K-blocks of the single-CTA variant's
// tile, and a 32 KB exchange instead of 96 KB (DSMEM moves ~20 B/cycle per SM, B300_MICROARCH).
template <int AMAJ, int BMAJ, int EPI>
__global__ void __launch_bounds__(NUM_THREADS, 1)
    tc_gemm_csplit2_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                           const __grid_constant__ CUtensorMap tmO, const __grid_constant__ CUtensorMap tmK, EpiArgs e,
                           int M, int N, int K) {
    constexpr int BN = 128;                   // pair tile columns
    using C = Cfg<BN / 2, EPI>;               // per CTA: A 128 x 64, B 64 x 64 per K-block
    constexpr int KS = 2;                     // K-blocks per ring stage
    constexpr int NST = C::STAGES / KS;       // ring stages
    constexpr int W = 64;                     // output columns each CTA owns
    constexpr uint32_t SLICE = 128u * W * 4;  // 32 KB
    static_assert(2 * SLICE <= (uint32_t)C::STAGES * C::STAGE_BYTES, "exchange does not fit the ring");
    static_assert(C::STAGES % KS == 0, "ring");
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    uint8_t *epi_stg = smem + C::STAGES * C::STAGE_BYTES;
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem + C::STAGES * C::STAGE_BYTES + C::EPI_STG);
    uint64_t *full = bars, *empty = bars + C::STAGES, *tfull = bars + 2 * C::STAGES, *rbar = tfull + 1;
    uint64_t *mbar = rbar + 1;
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(mbar + 8);
    uint8_t *outbox = smem, *recv = smem + SLICE;

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) PROBE(0);
    uint32_t crank;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(crank));
    const uint32_t prank = crank & 1u, split = crank >> 1;
    const uint16_t pmask = (uint16_t)(3u << (crank & ~1u));  // this pair's CTAs
    const uint32_t other = crank ^ 2u;                         // same rows, other K half
    const int tile = blockIdx.x / 4;
    const int m_blocks = (M + 255) / 256;
    const int m0p = (tile % m_blocks) * 256, n0 = (tile / m_blocks) * BN;
    const int m0 = m0p + (int)prank * BM;
    const int kblocks = (K + BK - 1) / BK;
    const int kper = ((kblocks + 1) / 2 + KS - 1) / KS * KS;  // a whole number of stages
    const int kb0 = (int)split * kper, kb1 = min(kblocks, kb0 + kper);

    if (warp == 0 && lane == 0) {
        asm volatile("prefetch.tensormap [%0];" ::"l"(&tmA) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(&tmB) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(&tmO) : "memory");
        if (EPI == EPI_MASK) asm volatile("prefetch.tensormap [%0];" ::"l"(&tmK) : "memory");
        for (int s = 0; s < NST; ++s) {
            mbar_init(smem_u32(&full[s]), 1);
            mbar_init(smem_u32(&empty[s]), 1);
        }
        mbar_init(smem_u32(tfull), 1);
        mbar_init(smem_u32(rbar), 1);
        for (int a = 0; a < 8; ++a) mbar_init(smem_u32(&mbar[a]), 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 2) {
        asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                     "r"(BN));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
    }
    tc_fence_before();
    cluster_sync_all();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;
    if (threadIdx.x == 0) PROBE(1);
    if (warp == 0 && lane == 0) mbar_expect_tx(smem_u32(rbar), SLICE);
    // programmatic dependent launch: the next GEMM of the chain may be scheduled now (it only
    // prefetches its weights before its own griddepcontrol.wait)
    if (threadIdx.x == 0) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");

    if (warp == 0) {
        if (lane == 0) {  // ===== TMA producer: this CTA's A rows and B half land on the leader's barrier
            int stage = 0;
            uint32_t phase = 0;
            auto load_a = [&](uint32_t sa, uint32_t fb, int k0) {
                if (AMAJ == KMAJ) {
                    tma_load_2d_cg<2>(sa, &tmA, fb, k0, m0);
                } else {
#pragma unroll
                    for (int j = 0; j < BM / 64; ++j) tma_load_2d_cg<2>(sa + j * BK * 128, &tmA, fb, m0 + 64 * j, k0);
                }
            };
            auto load_b = [&](uint32_t sb, uint32_t fb, int k0) {
                if (BMAJ == KMAJ) tma_load_2d_cg<2>(sb, &tmB, fb, k0, n0 + (int)prank * 64);
                else tma_load_2d_cg<2>(sb, &tmB, fb, n0 + (int)prank * 64, k0);
            };
            // prologue: the weights (B) of the first ring stages do not depend on the previous
            // kernel -- issue them before griddepcontrol.wait, the activations (A) after it
            const int npre = min(NST, (kb1 - kb0 + KS - 1) / KS);
            for (int st = 0; st < npre; ++st) {
                const uint32_t fb = smem_u32(&full[st]) & 0xFEFFFFFFu;
                const int kb = kb0 + st * KS, nk = min(KS, kb1 - kb);
                if (prank == 0) mbar_expect_tx(fb, 2 * nk * C::STAGE_BYTES);
                for (int h = 0; h < nk; ++h)
                    load_b(smem_u32(smem + (st * KS + h) * C::STAGE_BYTES) + C::A_BYTES, fb, (kb + h) * BK);
            }
            asm volatile("griddepcontrol.wait;" ::: "memory");
            for (int st = 0; st < npre; ++st) {
                const uint32_t fb = smem_u32(&full[st]) & 0xFEFFFFFFu;
                const int kb = kb0 + st * KS, nk = min(KS, kb1 - kb);
                for (int h = 0; h < nk; ++h) load_a(smem_u32(smem + (st * KS + h) * C::STAGE_BYTES), fb, (kb + h) * BK);
            }
            stage = npre % NST;
            phase = npre == NST ? 1u : 0u;
            for (int kb = kb0 + npre * KS; kb < kb1; kb += KS) {
                mbar_wait(smem_u32(&empty[stage]), phase ^ 1);
                const uint32_t fb = smem_u32(&full[stage]) & 0xFEFFFFFFu;
                const int nk = min(KS, kb1 - kb);
                if (prank == 0) mbar_expect_tx(fb, 2 * nk * C::STAGE_BYTES);
                for (int h = 0; h < nk; ++h) {
                    const uint32_t sa = smem_u32(smem + (stage * KS + h) * C::STAGE_BYTES);
                    load_a(sa, fb, (kb + h) * BK);
                    load_b(sa + C::A_BYTES, fb, (kb + h) * BK);
                }
                if (++stage == NST) { stage = 0; phase ^= 1; }
            }
        }
    } else if (warp == 1) {
        if (lane == 0 && prank == 0) {  // ===== MMA issuer (pair leader): M = 256, N = 128
            constexpr uint32_t idesc = make_idesc(2 * BM, BN, AMAJ, BMAJ);
            int stage = 0;
            uint32_t phase = 0;
            for (int kb = kb0; kb < kb1; kb += KS) {
                mbar_wait(smem_u32(&full[stage]), phase);
                tc_fence_after();
                if (kb == kb0) PROBE(3);
                const int nk = min(KS, kb1 - kb);
                for (int h = 0; h < nk; ++h) {
                    const uint32_t sa = smem_u32(smem + (stage * KS + h) * C::STAGE_BYTES), sb = sa + C::A_BYTES;
#pragma unroll
                    for (int k = 0; k < BK / UMMA_K; ++k) {
                        const uint64_t ad = AMAJ == KMAJ ? smem_desc(sa + k * 32, 16, 1024) : smem_desc(sa + k * 2048, BK * 128, 1024);
                        const uint64_t bd = BMAJ == KMAJ ? smem_desc(sb + k * 32, 16, 1024) : smem_desc(sb + k * 2048, BK * 128, 1024);
                        tc_mma_cg<2>(tmem_base, ad, bd, idesc, (kb > kb0 || h > 0 || k > 0) ? 1u : 0u);
                    }
                }
                tc_commit_cg<2>(smem_u32(&empty[stage]), pmask);
                if (++stage == NST) { stage = 0; phase ^= 1; }
            }
            PROBE(4);
            tc_commit_cg<2>(smem_u32(tfull), pmask);
        }
    } else if (warp >= 4) {
        mbar_wait(smem_u32(tfull), 0);
        tc_fence_after();
        if (warp == 4 && lane == 0) PROBE(5);
    }
    tc_fence_before();
    cluster_sync_all();  // both pairs' MMAs are complete: the rings are free for the exchange
    tc_fence_after();

    if (warp >= 4) {
        if (warp == 4 && lane == 0) PROBE(7);
        const int q = warp & 3;
        const int row = q * 32 + lane;
        const uint32_t tl = tmem_base + ((uint32_t)(q * 32) << 16);
        auto slice_off = [&](int col) {
            return (uint32_t)row * (W * 4) + (uint32_t)(((col >> 2) ^ (row & 15)) << 4);
        };
        const int mine = (int)split * W, theirs = W - mine;  // column offsets inside the pair tile
#pragma unroll 1
        for (int c = 0; c < W / 32; ++c) {
            float v[32];
            tmem_ld32(tl + theirs + c * 32, v);
#pragma unroll
            for (int i = 0; i < 8; ++i)
                st_shared_v4(smem_u32(outbox) + slice_off(c * 32 + 4 * i), v[4 * i], v[4 * i + 1], v[4 * i + 2],
                             v[4 * i + 3]);
        }
        fence_proxy_async();
        asm volatile("bar.sync 1, 128;" ::: "memory");
        if (warp == 4 && lane == 0) {
            asm volatile(
                "cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                    mapa_cluster(smem_u32(recv), other)),
                "r"(smem_u32(outbox)), "r"(SLICE), "r"(mapa_cluster(smem_u32(rbar), other))
                : "memory");
            PROBE(8);
        }
        uint8_t *wst = epi_stg + q * C::WARP_STG;
        const int r0 = m0 + q * 32;
        const int nc = n0 + mine;
        // own partials first (they do not wait for the exchange)
        float acc[W / 32][32];
#pragma unroll
        for (int c = 0; c < W / 32; ++c) tmem_ld32(tl + mine + c * 32, acc[c]);
        if (EPI == EPI_MASK && lane == 0) {
#pragma unroll
            for (int c = 0; c < W / 32; ++c) {
                mbar_expect_tx(smem_u32(&mbar[q * 2 + c]), 2048);
                tma_load_2d(smem_u32(wst + 2 * C::OUT_TILE + c * 2048), &tmK, smem_u32(&mbar[q * 2 + c]), nc + c * 32, r0);
            }
        }
        // the bias of the owned columns, loaded (16-byte vectors) while the exchange is in flight
        float bv[W / 32][32];
#pragma unroll
        for (int c = 0; c < W / 32; ++c)
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                const int col = nc + c * 32 + 4 * i;
                float4 x = make_float4(0.f, 0.f, 0.f, 0.f);
                if (EPI == EPI_STORE && e.bias && col + 4 <= N) x = __ldg(reinterpret_cast<const float4 *>(e.bias + col));
                else if (EPI == EPI_STORE && e.bias)
                    for (int j = 0; j < 4 && col + j < N; ++j) (&x.x)[j] = __ldg(e.bias + col + j);
                bv[c][4 * i] = x.x, bv[c][4 * i + 1] = x.y, bv[c][4 * i + 2] = x.z, bv[c][4 * i + 3] = x.w;
            }
        EpiArgs en = e;
        en.bias = nullptr;  // added here
        mbar_wait(smem_u32(rbar), 0);
        if (warp == 4 && lane == 0) PROBE(9);
#pragma unroll
        for (int c = 0; c < W / 32; ++c) {
            const int col = nc + c * 32;
            float v[32];
            // the two K halves' partials (one fp32 addition: commutative, deterministic)
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                const float4 x = *reinterpret_cast<const float4 *>(recv + slice_off(c * 32 + 4 * i));
                v[4 * i] = acc[c][4 * i] + x.x, v[4 * i + 1] = acc[c][4 * i + 1] + x.y;
                v[4 * i + 2] = acc[c][4 * i + 2] + x.z, v[4 * i + 3] = acc[c][4 * i + 3] + x.w;
            }
            if (EPI == EPI_STORE && e.bias) {
#pragma unroll
                for (int i = 0; i < 32; ++i) v[i] += bv[c][i];
            }
            const uint8_t *mt = nullptr;
            if constexpr (EPI == EPI_MASK) {
                mbar_wait(smem_u32(&mbar[q * 2 + c]), 0);
                mt = wst + 2 * C::OUT_TILE + c * 2048;
            }
            epi_math<EPI>(en, v, r0 + lane, col, N, mt, lane);
            uint8_t *ot = wst + c * C::OUT_TILE;
            epi_stage<EPI>(ot, v, lane);
            fence_proxy_async();
            __syncwarp();
            if (lane == 0 && col < N) {
                tma_store_2d(&tmO, smem_u32(ot), col, r0);
                bulk_commit();
            }
        }
        if (lane == 0) bulk_wait_read0();  // (the stores complete with the grid)
        if (warp == 4 && lane == 0) PROBE(11);
    }
    tc_fence_before();
    cluster_sync_all();
    if (threadIdx.x == 0) PROBE(6);
    if (warp == 2) {
        tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(BN));
    }
}

// ---------------------------------------------------------------- RGB first conv layer, forward
// Packed-tap forward of a Cp = 8 input (the RGB layer: 3 channels padded to 8, 16 bytes per
// padded-grid pixel).  Output pixel m, tap t reads input row m + shift[t]; the 9 shifted
// 128-row windows of a tile are all inside ONE contiguous span of rows
// [m0 - (Wp+1), m0 + 128 + (Wp+1)), so a tile's whole A operand is one 1-D bulk copy of
// (128 + 2 (Wp+1)) x 16 B instead of 9 TMA boxes of 128 16-byte rows (the row count, not the
// bytes, bounded the box version: 566 us for 418 MB of output at 224^2, B = 64).  [px][8]
// bf16 IS the unswizzled K-major core-matrix layout (8 rows x 16 B), so tap t's operand is the
// span at row offset shift[t] + Wp + 1 -- two taps per K = 16 MMA, their distance as the
// descriptor's leading byte offset.  The weights W [Co][72] (+ a zero K = 72..79 slot) stay
// resident in shared memory for the whole persistent launch.
constexpr int C8_NS = 6;  // span ring depth
constexpr int C8_THREADS = 384;  // two epilogue groups of 4 warps: even / odd tiles (accumulator 0 / 1)
__global__ void __launch_bounds__(C8_THREADS, 1)
    conv_c8_fwd_kernel(const __grid_constant__ CUtensorMap tmB, const __grid_constant__ CUtensorMap tmO,
                       const __nv_bfloat16 *__restrict__ X, EpiArgs e, int M, int N, int span_bytes) {
    constexpr int BNW = 64;  // output channels (N <= 64)
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    uint8_t *sB = smem;                                   // 10 slots x 64 rows x 16 B
    uint8_t *ring = smem + 10 * 1024;                     // C8_NS spans
    uint8_t *epi_stg = ring + C8_NS * span_bytes;         // 8 warps x 2 x 2 KB (1024-aligned: span_bytes % 1024 == 0)
    uint64_t *bars = reinterpret_cast<uint64_t *>(epi_stg + 8 * 4096);
    uint64_t *full = bars, *empty = bars + C8_NS, *tfull = bars + 2 * C8_NS, *tempty = tfull + 2, *bbar = tempty + 2;
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(bbar + 1);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int Wp = e.conv.Wp, halo = Wp + 1;
    const int tiles = (M + BM - 1) / BM;

    if (warp == 0 && lane == 0) {
        asm volatile("prefetch.tensormap [%0];" ::"l"(&tmB) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(&tmO) : "memory");
        for (int s = 0; s < C8_NS; ++s) {
            mbar_init(smem_u32(&full[s]), 1);
            mbar_init(smem_u32(&empty[s]), 1);
        }
        for (int a = 0; a < 2; ++a) {
            mbar_init(smem_u32(&tfull[a]), 1);
            mbar_init(smem_u32(&tempty[a]), 4);
        }
        mbar_init(smem_u32(bbar), 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 2) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                     "r"(2 * BNW));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    // zero the span ring once: window rows a clipped copy leaves unwritten (the image's first /
    // last halo) then hold finite values -- they only feed border outputs, which are zeroed
    for (int i = threadIdx.x; i < C8_NS * span_bytes / 16; i += C8_THREADS)
        reinterpret_cast<uint4 *>(ring)[i] = make_uint4(0, 0, 0, 0);
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    if (warp == 0) {
        if (lane == 0) {  // ===== producer: the weights once, then one span per tile
            mbar_expect_tx(smem_u32(bbar), 10 * BNW * 16);
            for (int j = 0; j < 10; ++j) tma_load_2d(smem_u32(sB + j * 1024), &tmB, smem_u32(bbar), 8 * j, 0);
            int stage = 0;
            uint32_t phase = 0;
            for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
                mbar_wait(smem_u32(&empty[stage]), phase ^ 1);
                long r0 = (long)tile * BM - halo, r1 = (long)tile * BM + BM + halo;  // span rows [r0, r1)
                uint32_t dst = smem_u32(ring + stage * span_bytes);
                if (r0 < 0) { dst += (uint32_t)(-r0) * 16; r0 = 0; }
                if (r1 > M) r1 = M;
                const uint32_t bytes = (uint32_t)(r1 - r0) * 16;
                mbar_expect_tx(smem_u32(&full[stage]), bytes);
                asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                                 dst),
                             "l"(X + r0 * 8), "r"(bytes), "r"(smem_u32(&full[stage]))
                             : "memory");
                if (++stage == C8_NS) { stage = 0; phase ^= 1; }
            }
        }
    } else if (warp == 1) {
        if (lane == 0) {  // ===== MMA: K = 80 as 5 x K16, taps (2k, 2k+1); tap 9 = zero weights
            constexpr uint32_t idesc = make_idesc(BM, BNW, KMAJ, KMAJ);
            mbar_wait(smem_u32(bbar), 0);
            int off[10];
#pragma unroll
            for (int t = 0; t < 9; ++t) off[t] = (e.conv.a_shift[t] + halo) * 16;
            off[9] = off[8];  // (any finite rows: its weights are zero)
            int stage = 0, acc = 0;
            uint32_t phase = 0, acc_phase = 0;
            for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
                mbar_wait(smem_u32(&tempty[acc]), acc_phase ^ 1);
                mbar_wait(smem_u32(&full[stage]), phase);
                tc_fence_after();
                const uint32_t sp = smem_u32(ring + stage * span_bytes), sb = smem_u32(sB);
#pragma unroll
                for (int k = 0; k < 5; ++k) {
                    const uint64_t ad = smem_desc_ns(sp + off[2 * k], off[2 * k + 1] - off[2 * k], 128);
                    const uint64_t bd = smem_desc_ns(sb + 2 * k * 1024, 1024, 128);
                    tc_mma(tmem_base + acc * BNW, ad, bd, idesc, k > 0 ? 1u : 0u);
                }
                tc_commit(smem_u32(&empty[stage]));
                tc_commit(smem_u32(&tfull[acc]));
                if (++stage == C8_NS) { stage = 0; phase ^= 1; }
                if (++acc == 2) { acc = 0; acc_phase ^= 1; }
            }
        }
    } else if (warp >= 4) {  // ===== epilogue: bias + ReLU + zero border, bf16 TMA stores
        // group g = (warp - 4) / 4 takes this CTA's tiles of parity g (accumulator g): two tiles'
        // epilogues in flight, the epilogue (not the loads or the MMAs) bounds this kernel
        const int q = warp & 3, grp = (warp - 4) >> 2;
        uint8_t *wst = epi_stg + (warp - 4) * 4096;
        const int acc = grp;
        uint32_t acc_phase = 0, ocnt = 0;
        for (int tile = blockIdx.x + grp * gridDim.x; tile < tiles; tile += 2 * gridDim.x) {
            mbar_wait(smem_u32(&tfull[acc]), acc_phase);
            tc_fence_after();
            const int r0 = tile * BM + q * 32;
#pragma unroll 1
            for (int c = 0; c < BNW / 32 && c * 32 < N; ++c) {
                float v[32];
                tmem_ld32(tmem_base + ((uint32_t)(q * 32) << 16) + acc * BNW + c * 32, v);
                epi_math<EPI_STORE>(e, v, r0 + lane, c * 32, N, nullptr, lane);
                if (lane == 0) bulk_wait_read1();
                __syncwarp();
                uint8_t *ot = wst + (ocnt & 1) * 2048;
                epi_stage<EPI_STORE>(ot, v, lane);
                fence_proxy_async();
                __syncwarp();
                if (lane == 0) {
                    tma_store_2d(&tmO, smem_u32(ot), c * 32, r0);
                    bulk_commit();
                }
                ++ocnt;
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(smem_u32(&tempty[acc]));
            acc_phase ^= 1;
        }
        if (lane == 0) bulk_wait_read0();
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 2) {
        tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(2 * BNW));
    }
}

// ---------------------------------------------------------------- dW GEMM + fused optimizer update
// The weight-gradient GEMM of an unreplicated stage never leaves the chip: its accumulator
// tile is consumed in TMEM by the update, which reads the fp32 master tile (and Adam m, v),
// writes the new master and the new bf16 weight version.  That epilogue is pure HBM
// traffic (10 B/param for SGD, 26 B for Adam), so it is staged through shared memory with
// TMA: the producer warp prefetches the master (m, v) tile with cp.async.bulk.tensor into a
// 128B-swizzled buffer while the MMAs run, the epilogue warps update it in place (bank-
// conflict-free thanks to the swizzle) and one thread writes the tiles back with TMA bulk
// stores.  Everything moves as full lines with the TMA engine's queue depth instead of
// per-thread 16-byte accesses.
__device__ __forceinline__ void epi_bar() { asm volatile("bar.sync 1, 128;" ::: "memory"); }

// DEEP: 2 operand stages and 3 epilogue stages (more optimizer-state sub-tiles in flight per
// SM; the operands are L2 hits at K = 256)
template <int BN, bool ADAM, bool DEEP = false>
struct UpdCfg {
    static constexpr int A_BYTES = BM * BK * 2;
    static constexpr int B_BYTES = BN * BK * 2;
    static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
    static constexpr int STAGES = (BN == 256 || DEEP) ? 2 : 3;  // (BN 256: 2 x 48 KB operand stages fit beside the epilogue ring)
    // epilogue sub-tiles: ECOLS columns of the [128][BN] tile, double-buffered so the TMA
    // load of sub-tile k+1 and the TMA store of sub-tile k-1 overlap the update of k
    static constexpr int ECOLS = ADAM ? 32 : 64;
    static constexpr int ESTAGES = DEEP ? 3 : 2;
    static constexpr int NF32 = ADAM ? 3 : 1;           // master (+ m, v)
    static constexpr int F32_SUB = BM * ECOLS * 4;       // one fp32 sub-tile
    static constexpr int BF_SUB = BM * ECOLS * 2;        // one bf16 sub-tile
    static constexpr int EBUF = NF32 * F32_SUB + BF_SUB; // one epilogue stage
    static constexpr int TMEM_COLS = 2 * BN < 32 ? 32 : 2 * BN;
    static constexpr int SMEM = STAGES * STAGE_BYTES + ESTAGES * EBUF + 1024 + 256;
};

struct UpdArgs {
    float lr, b1, b2, eps, bc1, bc2;
};

template <int BN, int AMAJ, int BMAJ, bool ADAM, bool DEEP = false>
__global__ void __launch_bounds__(NUM_THREADS, 1)
    tc_gemm_update_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                          const __grid_constant__ CUtensorMap tmW, const __grid_constant__ CUtensorMap tmM,
                          const __grid_constant__ CUtensorMap tmV, const __grid_constant__ CUtensorMap tmS, UpdArgs u,
                          int M, int N, int K) {
    using C = UpdCfg<BN, ADAM, DEEP>;
    constexpr int SUBS = BN / C::ECOLS;        // epilogue sub-tiles per tile
    constexpr int F32_BOXES = C::ECOLS / 32;   // 32 fp32 = 128 B per swizzled box row
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    uint8_t *ebuf = smem + C::STAGES * C::STAGE_BYTES;
    uint64_t *bars = reinterpret_cast<uint64_t *>(ebuf + C::ESTAGES * C::EBUF);
    uint64_t *full = bars, *empty = bars + C::STAGES, *tfull = bars + 2 * C::STAGES, *tempty = tfull + 2;
    uint64_t *wfull = tempty + 2, *wempty = wfull + C::ESTAGES;
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(wempty + C::ESTAGES);

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int m_blocks = (M + BM - 1) / BM, n_blocks = (N + BN - 1) / BN;
    const int tiles = m_blocks * n_blocks;
    const int kblocks = (K + BK - 1) / BK;

    if (warp == 0 && lane == 0) {
        const CUtensorMap *maps[6] = {&tmA, &tmB, &tmW, &tmM, &tmV, &tmS};
        for (int i = 0; i < 6; ++i) asm volatile("prefetch.tensormap [%0];" ::"l"(maps[i]) : "memory");
        for (int s2 = 0; s2 < C::STAGES; ++s2) {
            mbar_init(smem_u32(&full[s2]), 1);
            mbar_init(smem_u32(&empty[s2]), 1);
        }
        for (int a = 0; a < 2; ++a) {
            mbar_init(smem_u32(&tfull[a]), 1);
            mbar_init(smem_u32(&tempty[a]), 4);
        }
        for (int e = 0; e < C::ESTAGES; ++e) {
            mbar_init(smem_u32(&wfull[e]), 1);
            mbar_init(smem_u32(&wempty[e]), 1);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 2) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                     "r"(C::TMEM_COLS));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    if (warp == 0) {
        if (lane == 0) {
            int stage = 0, es = 0;
            uint32_t phase = 0, ephase = 0;
            const CUtensorMap *fm[3] = {&tmW, &tmM, &tmV};
            for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
                const int m0 = (tile % m_blocks) * BM, n0 = (tile / m_blocks) * BN;
                for (int kb = 0; kb < kblocks; ++kb) {
                    mbar_wait(smem_u32(&empty[stage]), phase ^ 1);
                    const uint32_t fb = smem_u32(&full[stage]);
                    mbar_expect_tx(fb, C::STAGE_BYTES);
                    const uint32_t sa = smem_u32(smem + stage * C::STAGE_BYTES);
                    const uint32_t sb = sa + C::A_BYTES;
                    const int k0 = kb * BK;
                    if (AMAJ == KMAJ) tma_load_2d(sa, &tmA, fb, k0, m0);
                    else
#pragma unroll
                        for (int j = 0; j < BM / 64; ++j) tma_load_2d(sa + j * BK * 128, &tmA, fb, m0 + 64 * j, k0);
                    if (BMAJ == KMAJ) tma_load_2d(sb, &tmB, fb, k0, n0);
                    else
#pragma unroll
                        for (int j = 0; j < BN / 64; ++j) tma_load_2d(sb + j * BK * 128, &tmB, fb, n0 + 64 * j, k0);
                    if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
                }
                // optimizer-state sub-tiles of this output tile into the epilogue ring
                for (int sub = 0; sub < SUBS; ++sub) {
                    mbar_wait(smem_u32(&wempty[es]), ephase ^ 1);
                    const uint32_t wb = smem_u32(&wfull[es]);
                    mbar_expect_tx(wb, C::NF32 * C::F32_SUB);
                    uint8_t *buf = ebuf + es * C::EBUF;
#pragma unroll
                    for (int t3 = 0; t3 < C::NF32; ++t3)
#pragma unroll
                        for (int q = 0; q < F32_BOXES; ++q)
                            tma_load_2d(smem_u32(buf + t3 * C::F32_SUB + q * BM * 128), fm[t3], wb,
                                        n0 + sub * C::ECOLS + 32 * q, m0);
                    if (++es == C::ESTAGES) { es = 0; ephase ^= 1; }
                }
            }
        }
    } else if (warp == 1) {
        if (lane == 0) {
            constexpr uint32_t idesc = make_idesc(BM, BN, AMAJ, BMAJ);
            int stage = 0;
            uint32_t phase = 0;
            int acc = 0;
            uint32_t acc_phase = 0;
            for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
                mbar_wait(smem_u32(&tempty[acc]), acc_phase ^ 1);
                tc_fence_after();
                const uint32_t d = tmem_base + acc * BN;
                for (int kb = 0; kb < kblocks; ++kb) {
                    mbar_wait(smem_u32(&full[stage]), phase);
                    tc_fence_after();
                    const uint32_t sa = smem_u32(smem + stage * C::STAGE_BYTES);
                    const uint32_t sb = sa + C::A_BYTES;
#pragma unroll
                    for (int k = 0; k < BK / UMMA_K; ++k) {
                        const uint64_t ad = AMAJ == KMAJ ? smem_desc(sa + k * 32, 16, 1024)
                                                         : smem_desc(sa + k * 2048, BK * 128, 1024);
                        const uint64_t bd = BMAJ == KMAJ ? smem_desc(sb + k * 32, 16, 1024)
                                                         : smem_desc(sb + k * 2048, BK * 128, 1024);
                        tc_mma(d, ad, bd, idesc, (kb | k) != 0);
                    }
                    tc_commit(smem_u32(&empty[stage]));
                    if (++stage == C::STAGES) { stage = 0; phase ^= 1; }
                }
                tc_commit(smem_u32(&tfull[acc]));
                if (++acc == 2) { acc = 0; acc_phase ^= 1; }
            }
        }
    } else if (warp >= 4) {
        const int q4 = warp & 3;
        const int r = q4 * 32 + lane;  // tile row owned by this thread (TMEM lane)
        const uint32_t rsw = (uint32_t)(r & 7);
        const bool leader = (warp == 4 && lane == 0);
        int acc = 0, es = 0;
        uint32_t acc_phase = 0, ephase = 0;
        for (int tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
            const int m0 = (tile % m_blocks) * BM, n0 = (tile / m_blocks) * BN;
            mbar_wait(smem_u32(&tfull[acc]), acc_phase);
            tc_fence_after();
            for (int sub = 0; sub < SUBS; ++sub) {
                uint8_t *buf = ebuf + es * C::EBUF;
                uint8_t *bf_tile = buf + C::NF32 * C::F32_SUB;
                mbar_wait(smem_u32(&wfull[es]), ephase);
#pragma unroll 1
                for (int cc = 0; cc < C::ECOLS / 32; ++cc) {
                    float g[32];
                    tmem_ld32(tmem_base + ((uint32_t)(q4 * 32) << 16) + acc * BN + sub * C::ECOLS + cc * 32, g);
                    // fp32 box cc, row r: 16-byte chunk j lives at chunk (j ^ (r & 7))
                    float *wrow = reinterpret_cast<float *>(buf + cc * BM * 128 + r * 128);
                    float *mrow = reinterpret_cast<float *>(buf + C::F32_SUB + cc * BM * 128 + r * 128);
                    float *vrow = reinterpret_cast<float *>(buf + 2 * C::F32_SUB + cc * BM * 128 + r * 128);
                    uint32_t packed[16];
#pragma unroll
                    for (int j = 0; j < 8; ++j) {
                        const int pj = (int)((uint32_t)j ^ rsw) * 4;
                        float4 w4 = *reinterpret_cast<float4 *>(wrow + pj);
                        float wv[4] = {w4.x, w4.y, w4.z, w4.w};
                        if constexpr (ADAM) {
                            float4 m4 = *reinterpret_cast<float4 *>(mrow + pj);
                            float4 v4 = *reinterpret_cast<float4 *>(vrow + pj);
                            float mm[4] = {m4.x, m4.y, m4.z, m4.w}, vv[4] = {v4.x, v4.y, v4.z, v4.w};
#pragma unroll
                            for (int i = 0; i < 4; ++i) {
                                const float gi = g[j * 4 + i];
                                mm[i] = u.b1 * mm[i] + (1.f - u.b1) * gi;
                                vv[i] = u.b2 * vv[i] + (1.f - u.b2) * gi * gi;
                                wv[i] = wv[i] - u.lr * (mm[i] / u.bc1) / (sqrtf(vv[i] / u.bc2) + u.eps);
                            }
                            *reinterpret_cast<float4 *>(mrow + pj) = make_float4(mm[0], mm[1], mm[2], mm[3]);
                            *reinterpret_cast<float4 *>(vrow + pj) = make_float4(vv[0], vv[1], vv[2], vv[3]);
                        } else {
#pragma unroll
                            for (int i = 0; i < 4; ++i) wv[i] = wv[i] - u.lr * g[j * 4 + i];
                        }
                        *reinterpret_cast<float4 *>(wrow + pj) = make_float4(wv[0], wv[1], wv[2], wv[3]);
                        packed[j * 2] = pack_bf16(wv[0], wv[1]);
                        packed[j * 2 + 1] = pack_bf16(wv[2], wv[3]);
                    }
                    // bf16 sub-tile: one 64-column box when ECOLS = 64, a 32-column box otherwise
                    constexpr int BF_ROW = C::ECOLS * 2;  // bytes per bf16 row of the sub-tile box
                    uint8_t *brow = bf_tile + r * BF_ROW;
#pragma unroll
                    for (int u4 = 0; u4 < 4; ++u4) {
                        const uint32_t lj = (uint32_t)(cc * 4 + u4);
                        const uint32_t pjb = BF_ROW == 128 ? (lj ^ rsw) : (lj ^ ((rsw >> 1) & 3));
                        *reinterpret_cast<uint4 *>(brow + (pjb << 4)) =
                            make_uint4(packed[u4 * 4], packed[u4 * 4 + 1], packed[u4 * 4 + 2], packed[u4 * 4 + 3]);
                    }
                }
                if (sub == SUBS - 1) {
                    // accumulator fully consumed: hand TMEM back to the MMA warp
                    tc_fence_before();
                    __syncwarp();
                    if (lane == 0) mbar_arrive(smem_u32(&tempty[acc]));
                }
                fence_proxy_async();
                epi_bar();
                if (leader) {
                    const CUtensorMap *fm[3] = {&tmW, &tmM, &tmV};
                    const int c0 = n0 + sub * C::ECOLS;
#pragma unroll
                    for (int t3 = 0; t3 < C::NF32; ++t3)
#pragma unroll
                        for (int q = 0; q < F32_BOXES; ++q)
                            tma_store_2d(fm[t3], smem_u32(buf + t3 * C::F32_SUB + q * BM * 128), c0 + 32 * q, m0);
                    tma_store_2d(&tmS, smem_u32(bf_tile), c0, m0);
                    bulk_commit();
                    // the bulk store reads shared memory quickly; once it has, the buffer can
                    // take the next sub-tile's load while the global writes drain
                    bulk_wait_read0();
                    mbar_arrive(smem_u32(&wempty[es]));
                }
                if (++es == C::ESTAGES) { es = 0; ephase ^= 1; }
            }
            if (++acc == 2) { acc = 0; acc_phase ^= 1; }
        }
        if (leader) bulk_wait0();
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 2) {
        tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(C::TMEM_COLS));
    }
}

// ---------------------------------------------------------------- host side
struct MapKey {
    const void *base;
    long inner, outer, ld;
    int bi, bo, f32, sw;
    long planes = 0;  // 3-D maps: number of [outer][inner] planes (plane stride outer*ld)
    bool operator==(const MapKey &o) const {
        return base == o.base && inner == o.inner && outer == o.outer && ld == o.ld && bi == o.bi && bo == o.bo &&
               f32 == o.f32 && sw == o.sw && planes == o.planes;
    }
};
struct MapKeyHash {
    size_t operator()(const MapKey &k) const {
        size_t h = std::hash<const void *>()(k.base);
        for (long v : {k.inner, k.outer, k.ld, (long)k.bi, (long)k.bo, (long)(k.f32 * 1024 + k.sw), k.planes})
            h = h * 1000003u ^ std::hash<long>()(v);
        return h;
    }
};

bool encode_map(CUtensorMap *map, const void *base, long inner, long outer, long ld_elems, int box_inner,
                int box_outer, bool f32, int swizzle_bytes);
bool make_map3_f32(CUtensorMap *map, const void *base, long inner, long outer, long ld_elems, long planes,
                   int box_inner, int box_outer, int swizzle_bytes);

// Tensor maps are encoded once per (buffer, shape, box) and reused: encoding costs a driver
// call on every launch otherwise, and the runtime's buffers are stable for a context's life.
bool make_map(CUtensorMap *map, const void *base, long inner, long outer, long ld_elems, int box_inner, int box_outer,
              bool f32 = false, int swizzle_bytes = 128) {
    thread_local std::unordered_map<MapKey, CUtensorMap, MapKeyHash> cache;
    const MapKey key{base, inner, outer, ld_elems, box_inner, box_outer, (int)f32, swizzle_bytes};
    auto it = cache.find(key);
    if (it != cache.end()) {
        *map = it->second;
        return true;
    }
    if (!encode_map(map, base, inner, outer, ld_elems, box_inner, box_outer, f32, swizzle_bytes)) return false;
    if (cache.size() > 65536) cache.clear();
    cache.emplace(key, *map);
    return true;
}

// 3-D fp32 map over `planes` stacked [outer][inner] matrices (split-K partials: one plane per
// split, so a tile's out-of-range rows are clipped at its own split's M, not the next split's)
bool make_map3_f32(CUtensorMap *map, const void *base, long inner, long outer, long ld_elems, long planes,
                   int box_inner, int box_outer, int swizzle_bytes) {
    thread_local std::unordered_map<MapKey, CUtensorMap, MapKeyHash> cache;
    MapKey key{base, inner, outer, ld_elems, box_inner, box_outer, 1, swizzle_bytes};
    key.planes = planes;
    auto it = cache.find(key);
    if (it != cache.end()) {
        *map = it->second;
        return true;
    }
    const Driver *d = driver();
    if (!d) return false;
    cuuint64_t dims[3] = {(cuuint64_t)inner, (cuuint64_t)outer, (cuuint64_t)planes};
    cuuint64_t strides[2] = {(cuuint64_t)ld_elems * 4, (cuuint64_t)ld_elems * 4 * outer};
    cuuint32_t box[3] = {(cuuint32_t)box_inner, (cuuint32_t)box_outer, 1};
    cuuint32_t estr[3] = {1, 1, 1};
    CUresult r = d->tensorMapEncodeTiled(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, const_cast<void *>(base), dims,
                                         strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                                         swizzle_bytes == 128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE,
                                         CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return false;
    if (cache.size() > 65536) cache.clear();
    cache.emplace(key, *map);
    return true;
}

bool encode_map(CUtensorMap *map, const void *base, long inner, long outer, long ld_elems, int box_inner,
                int box_outer, bool f32, int swizzle_bytes) {
    const Driver *d = driver();
    if (!d) return false;
    cuuint64_t dims[2] = {(cuuint64_t)inner, (cuuint64_t)outer};
    cuuint64_t strides[1] = {(cuuint64_t)ld_elems * (f32 ? 4 : 2)};
    cuuint32_t box[2] = {(cuuint32_t)box_inner, (cuuint32_t)box_outer};
    cuuint32_t estr[2] = {1, 1};
    CUresult r = d->tensorMapEncodeTiled(map, f32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_BFLOAT16,
                                         2, const_cast<void *>(base), dims,
                                         strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                                         swizzle_bytes == 64    ? CU_TENSOR_MAP_SWIZZLE_64B
                                         : swizzle_bytes == 0 ? CU_TENSOR_MAP_SWIZZLE_NONE
                                                              : CU_TENSOR_MAP_SWIZZLE_128B,
                                         CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                                         CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
}

int num_sms() {
    static int n = 0;
    if (!n) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        if (n <= 0) n = 148;
    }
    return n;
}

// tools only: PD_GEMM_PROBE=<file> appends one line per launch with each CTA's phase stamps
// (ns since the earliest kernel-entry stamp): entry, setup done, first TMA issued, first stage
// full, second stage full, last MMA issued, accumulator ready, epilogue done
static unsigned long long *probe_buf() {
    static unsigned long long *p = nullptr;
    static bool init = false;
    if (!init) {
        init = true;
        if (getenv("PD_GEMM_PROBE") && cudaMalloc(&p, 1024 * 16 * sizeof(unsigned long long)) != cudaSuccess) p = nullptr;
        if (p) cudaMemset(p, 0, 1024 * 16 * sizeof(unsigned long long));
    }
    return p;
}
static void probe_dump(int grid, const Gemm &g, int bn, int cg, int ksplit) {
    unsigned long long *p = probe_buf();
    if (!p) return;
    std::vector<unsigned long long> h((size_t)grid * 16);
    cudaDeviceSynchronize();
    cudaMemcpy(h.data(), p, h.size() * 8, cudaMemcpyDeviceToHost);
    unsigned long long t0 = ~0ull;
    for (int b = 0; b < grid; ++b) t0 = std::min(t0, h[b * 16]);
    FILE *f = fopen(getenv("PD_GEMM_PROBE"), "a");
    if (!f) return;
    fprintf(f, "M=%d N=%d K=%d BN=%d CG=%d S=%d grid=%d", g.M, g.N, g.K, bn, cg, ksplit, grid);
    const int order[12] = {0, 1, 2, 3, 7, 4, 5, 8, 9, 10, 11, 6};
    for (int b = 0; b < grid; ++b) {
        fprintf(f, " |");
        for (int i : order) fprintf(f, " %lld", h[b * 16 + i] ? (long long)(h[b * 16 + i] - t0) : -1LL);
    }
    fprintf(f, "\n");
    fclose(f);
    cudaMemset(p, 0, 1024 * 16 * sizeof(unsigned long long));
}

template <int BN, int AMAJ, int BMAJ, int EPI, int CG>
cudaError_t launch(const Gemm &g, const CUtensorMap &ma, const CUtensorMap &mb, const EpiArgs &e0, cudaStream_t s) {
    using C = Cfg<BN / CG, EPI>;
    EpiArgs e = e0;
    e.probe = probe_buf();
    auto kern = tc_gemm_kernel<BN, AMAJ, BMAJ, EPI, CG>;
    static bool attr_set = false;  // per instantiation; benign race (idempotent)
    if (!attr_set) {
        cudaError_t err = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
        if (err != cudaSuccess) return err;
        attr_set = true;
    }
    // epilogue tensor maps: output tile {32 cols, 32 rows} (bf16 64B-swizzled / fp32 128B-swizzled;
    // split-K partials stacked as [S*M][N]) and the ReLU-mask tile
    CUtensorMap mo = ma, mk = ma;
    if (EPI == EPI_STORE || EPI == EPI_MASK) {
        if (!make_map(&mo, e.out, g.N, g.M, e.ldo, 32, 32, false, 64)) return cudaErrorInvalidValue;
        if (EPI == EPI_MASK && !make_map(&mk, e.mask, g.N, g.M, e.ldm, 32, 32, false, 64))
            return cudaErrorInvalidValue;
    } else if (EPI == EPI_F32) {
        if (!e.atomic_out && e.split_stride) {
            if (e.split_stride != (long)g.M * e.ldo ||
                !make_map3_f32(&mo, e.out, g.N, g.M, e.ldo, e.ksplit, 32, 32, 128))
                return cudaErrorInvalidValue;
        } else if (!make_map(&mo, e.out, g.N, g.M, e.ldo, 32, 32, true, 128)) {
            return cudaErrorInvalidValue;
        }
    }
    const int units = ((g.M + BM * CG - 1) / (BM * CG)) * ((g.N + BN - 1) / BN) * e.ksplit;
    int slots = num_sms() / CG;
    if (g.max_ctas > 0 && g.max_ctas / CG < slots) slots = g.max_ctas / CG > 0 ? g.max_ctas / CG : 1;
    const int grid = CG * (units < slots ? units : slots);
    const int cluster = CG;
    if (cluster == 1) {
        kern<<<grid, NUM_THREADS, C::SMEM, s>>>(ma, mb, mo, mk, e, g.M, g.N, g.K);
    } else {
        cudaLaunchConfig_t cfg{};
        cfg.gridDim = dim3(grid);
        cfg.blockDim = dim3(NUM_THREADS);
        cfg.dynamicSmemBytes = C::SMEM;
        cfg.stream = s;
        cudaLaunchAttribute attr[1];
        attr[0].id = cudaLaunchAttributeClusterDimension;
        attr[0].val.clusterDim.x = cluster;
        attr[0].val.clusterDim.y = 1;
        attr[0].val.clusterDim.z = 1;
        cfg.attrs = attr;
        cfg.numAttrs = 1;
        cudaError_t err = cudaLaunchKernelEx(&cfg, kern, ma, mb, mo, mk, e, g.M, g.N, g.K);
        if (err != cudaSuccess) return err;
    }
    if (e.probe) probe_dump(grid, g, BN, CG, e.ksplit);
    ++tl_launches;
    return cudaGetLastError();
}

template <int BN, int AMAJ, int BMAJ, int CG>
cudaError_t dispatch_epi(const Gemm &g, const CUtensorMap &ma, const CUtensorMap &mb, const EpiArgs &e,
                         cudaStream_t s) {
    switch (g.epi) {
    case EPI_STORE: return launch<BN, AMAJ, BMAJ, EPI_STORE, CG>(g, ma, mb, e, s);
    case EPI_MASK: return launch<BN, AMAJ, BMAJ, EPI_MASK, CG>(g, ma, mb, e, s);
    case EPI_F32: return launch<BN, AMAJ, BMAJ, EPI_F32, CG>(g, ma, mb, e, s);
    case EPI_SGD: return launch<BN, AMAJ, BMAJ, EPI_SGD, 1>(g, ma, mb, e, s);
    case EPI_ADAM: return launch<BN, AMAJ, BMAJ, EPI_ADAM, 1>(g, ma, mb, e, s);
    }
    return cudaErrorInvalidValue;
}

template <int BN, int CG = 1>
cudaError_t dispatch_major(const Gemm &g, const CUtensorMap &ma, const CUtensorMap &mb, const EpiArgs &e,
                           cudaStream_t s) {
    if (g.amaj == KMAJ && g.bmaj == KMAJ) return dispatch_epi<BN, KMAJ, KMAJ, CG>(g, ma, mb, e, s);
    if (g.amaj == KMAJ && g.bmaj == MNMAJ) return dispatch_epi<BN, KMAJ, MNMAJ, CG>(g, ma, mb, e, s);
    if (g.amaj == MNMAJ && g.bmaj == MNMAJ) return dispatch_epi<BN, MNMAJ, MNMAJ, CG>(g, ma, mb, e, s);
    return dispatch_epi<BN, MNMAJ, KMAJ, CG>(g, ma, mb, e, s);
}

// cluster split-K launch: grid = tiles x S CTAs, clusters of S (the K-splits of one tile)
template <int AMAJ, int BMAJ, int EPI, int S>
cudaError_t launch_csplit(const Gemm &g, const CUtensorMap &ma, const CUtensorMap &mb, const EpiArgs &e,
                          cudaStream_t s) {
    using C = Cfg<256, EPI>;
    auto kern = tc_gemm_csplit_kernel<AMAJ, BMAJ, EPI, S>;
    static bool attr_set = false;
    if (!attr_set) {
        cudaError_t err = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
        if (err != cudaSuccess) return err;
        attr_set = true;
    }
    CUtensorMap mo = ma, mk = ma;
    if (!make_map(&mo, e.out, g.N, g.M, e.ldo, 32, 32, false, 64)) return cudaErrorInvalidValue;
    if (EPI == EPI_MASK && !make_map(&mk, e.mask, g.N, g.M, e.ldm, 32, 32, false, 64)) return cudaErrorInvalidValue;
    const int tiles = ((g.M + BM - 1) / BM) * ((g.N + 255) / 256);
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(tiles * S);
    cfg.blockDim = dim3(NUM_THREADS);
    cfg.dynamicSmemBytes = C::SMEM;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = S;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    EpiArgs ep = e;
    ep.probe = probe_buf();
    cudaError_t err = cudaLaunchKernelEx(&cfg, kern, ma, mb, mo, mk, ep, g.M, g.N, g.K);
    if (err != cudaSuccess) return err;
    if (ep.probe) probe_dump(tiles * S, g, 256, -S, S);  // CG = -S marks the cluster split-K kernel
    ++tl_launches;
    return cudaGetLastError();
}

template <int AMAJ, int BMAJ, int EPI>
cudaError_t launch_csplit2(const Gemm &g, const CUtensorMap &ma, const CUtensorMap &mb, const EpiArgs &e,
                           cudaStream_t s) {
    using C = Cfg<64, EPI>;
    auto kern = tc_gemm_csplit2_kernel<AMAJ, BMAJ, EPI>;
    static bool attr_set = false;
    if (!attr_set) {
        cudaError_t err = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
        if (err != cudaSuccess) return err;
        attr_set = true;
    }
    CUtensorMap mo = ma, mk = ma;
    if (!make_map(&mo, e.out, g.N, g.M, e.ldo, 32, 32, false, 64)) return cudaErrorInvalidValue;
    if (EPI == EPI_MASK && !make_map(&mk, e.mask, g.N, g.M, e.ldm, 32, 32, false, 64)) return cudaErrorInvalidValue;
    const int tiles = ((g.M + 255) / 256) * ((g.N + 127) / 128);
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(tiles * 4);
    cfg.blockDim = dim3(NUM_THREADS);
    cfg.dynamicSmemBytes = C::SMEM;
    cfg.stream = s;
    cudaLaunchAttribute attr[2];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = 4;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[1].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = g.pdl ? 2 : 1;  // (measured: MLP-4096 234.3k -> 239.5k samples/s)
    EpiArgs ep = e;
    ep.probe = probe_buf();
    cudaError_t err = cudaLaunchKernelEx(&cfg, kern, ma, mb, mo, mk, ep, g.M, g.N, g.K);
    if (err != cudaSuccess) return err;
    if (ep.probe) probe_dump(tiles * 4, g, 128, -2, 2);
    ++tl_launches;
    return cudaGetLastError();
}

template <int EPI, int S>
cudaError_t csplit_major(const Gemm &g, const CUtensorMap &ma, const CUtensorMap &mb, const EpiArgs &e, cudaStream_t s) {
    if (g.amaj == KMAJ && g.bmaj == KMAJ) return launch_csplit<KMAJ, KMAJ, EPI, S>(g, ma, mb, e, s);
    if (g.amaj == KMAJ && g.bmaj == MNMAJ) return launch_csplit<KMAJ, MNMAJ, EPI, S>(g, ma, mb, e, s);
    return cudaErrorInvalidValue;
}

template <int BN, int AMAJ, int BMAJ, bool ADAM, bool DEEP = false>
cudaError_t launch_update(const Gemm &g, const CUtensorMap &ma, const CUtensorMap &mb, const CUtensorMap &mw,
                          const CUtensorMap &mm, const CUtensorMap &mv, const CUtensorMap &ms, const UpdArgs &u,
                          cudaStream_t s) {
    using C = UpdCfg<BN, ADAM, DEEP>;
    auto kern = tc_gemm_update_kernel<BN, AMAJ, BMAJ, ADAM, DEEP>;
    static bool attr_set = false;
    if (!attr_set) {
        cudaError_t err = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
        if (err != cudaSuccess) return err;
        attr_set = true;
    }
    const int tiles = ((g.M + BM - 1) / BM) * ((g.N + BN - 1) / BN);
    const int cap = g.max_ctas > 0 && g.max_ctas < num_sms() ? g.max_ctas : num_sms();
    const int grid = tiles < cap ? tiles : cap;
    kern<<<grid, NUM_THREADS, C::SMEM, s>>>(ma, mb, mw, mm, mv, ms, u, g.M, g.N, g.K);
    ++tl_launches;
    return cudaGetLastError();
}

template <int BN, bool ADAM>
cudaError_t update_major(const Gemm &g, const CUtensorMap &ma, const CUtensorMap &mb, const CUtensorMap &mw,
                         const CUtensorMap &mm, const CUtensorMap &mv, const CUtensorMap &ms, const UpdArgs &u,
                         cudaStream_t s) {
    // SGD dW layout: the deeper epilogue ring by default (measured: 42 -> 40 us isolated, MLP-4096
    // step +3 %); PD_UPD_DEEP=0 for the 3 + 2 stage variant (read per call)
    const char *dp = getenv("PD_UPD_DEEP");
    if (g.amaj == MNMAJ && g.bmaj == MNMAJ && !ADAM && BN == 128 && !(dp && atoi(dp) == 0))
        return launch_update<BN, MNMAJ, MNMAJ, ADAM, true>(g, ma, mb, mw, mm, mv, ms, u, s);
    if (g.amaj == MNMAJ && g.bmaj == MNMAJ) return launch_update<BN, MNMAJ, MNMAJ, ADAM>(g, ma, mb, mw, mm, mv, ms, u, s);
    if (g.amaj == KMAJ && g.bmaj == KMAJ) return launch_update<BN, KMAJ, KMAJ, ADAM>(g, ma, mb, mw, mm, mv, ms, u, s);
    if (g.amaj == KMAJ) return launch_update<BN, KMAJ, MNMAJ, ADAM>(g, ma, mb, mw, mm, mv, ms, u, s);
    return launch_update<BN, MNMAJ, KMAJ, ADAM>(g, ma, mb, mw, mm, mv, ms, u, s);
}

// dW GEMM with the optimizer update fused (TMA-staged epilogue).  Requirements: ldo == N
// rows 16-byte aligned (N % 8 == 0 for bf16, % 4 for fp32).
cudaError_t gemm_bf16_update(const Gemm &g, cudaStream_t s) {
    const bool adam = g.epi == EPI_ADAM;
    // tile width: the update streams master (+ Adam m, v) per output element, the GEMM streams
    // (128 + BN) x 64 operand elements per K-block into the SM; wider tiles raise the FLOPs per
    // ingested byte (the per-SM TMA ingest, ~60 GB/s, bounds these tiles -- tools/tma_bw.cu)
    constexpr int bn_adam = 128;
    const char *bs = getenv("PD_UPD_BN_SGD");  // read per call (tests toggle it)
    const int bn_sgd = bs && atoi(bs) == 256 ? 256 : 128;
    const int BN = adam ? bn_adam : bn_sgd;
    CUtensorMap ma, mbm, mw, mm, mv, ms;
    const bool okA = g.amaj == KMAJ ? make_map(&ma, g.A, g.K, g.M, g.lda, 64, BM)
                                    : make_map(&ma, g.A, g.M, g.K, g.lda, 64, BK);
    const bool okB = g.bmaj == KMAJ ? make_map(&mbm, g.B, g.K, g.N, g.ldb, 64, BN)
                                    : make_map(&mbm, g.B, g.N, g.K, g.ldb, 64, BK);
    const int ecols = adam ? 32 : 64;  // UpdCfg::ECOLS
    bool ok = okA && okB && make_map(&mw, g.master, g.N, g.M, g.ldo, 32, BM, true) &&
              make_map(&ms, g.slot, g.N, g.M, g.ldo, ecols, BM, false, ecols == 64 ? 128 : 64);
    if (adam) ok = ok && make_map(&mm, g.adam_m, g.N, g.M, g.ldo, 32, BM, true) &&
                   make_map(&mv, g.adam_v, g.N, g.M, g.ldo, 32, BM, true);
    else mm = mv = mw;
    if (!ok) return cudaErrorInvalidValue;
    UpdArgs u{g.lr, g.b1, g.b2, g.eps, 1.f - powf(g.b1, (float)g.step), 1.f - powf(g.b2, (float)g.step)};
    if (adam) return BN == 64 ? update_major<64, true>(g, ma, mbm, mw, mm, mv, ms, u, s)
                              : update_major<128, true>(g, ma, mbm, mw, mm, mv, ms, u, s);
    return BN == 256 ? update_major<256, false>(g, ma, mbm, mw, mm, mv, ms, u, s)
                     : update_major<128, false>(g, ma, mbm, mw, mm, mv, ms, u, s);
}

// out = act(sum_s ws[s] + bias) or (sum_s ws[s]) * (mask > 0), bf16; partials summed in
// split order (deterministic).  4 columns per thread, 16-byte loads.
__global__ void splitk_epilogue_kernel(const float *ws, int S, long split_stride, int M, int N,
                                       const float *__restrict__ bias, int relu, const __nv_bfloat16 *__restrict__ mask,
                                       long ldm, __nv_bfloat16 *__restrict__ out, long ldo,
                                       float *__restrict__ zero_ws) {
    const long n4 = N / 4;
    const long total = (long)M * n4;
    for (long i = (long)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (long)gridDim.x * blockDim.x) {
        const long m = i / n4, c = (i % n4) * 4;
        float4 a = *reinterpret_cast<const float4 *>(ws + m * N + c);
        if (zero_ws) *reinterpret_cast<float4 *>(zero_ws + m * N + c) = make_float4(0.f, 0.f, 0.f, 0.f);
        for (int sp = 1; sp < S; ++sp) {
            const float4 b = *reinterpret_cast<const float4 *>(ws + sp * split_stride + m * N + c);
            a.x += b.x; a.y += b.y; a.z += b.z; a.w += b.w;
        }
        float v[4] = {a.x, a.y, a.z, a.w};
        if (bias) {
#pragma unroll
            for (int j = 0; j < 4; ++j) v[j] += bias[c + j];
        }
        if (relu) {
#pragma unroll
            for (int j = 0; j < 4; ++j) v[j] = fmaxf(v[j], 0.f);
        }
        if (mask) {
            const uint2 mr = *reinterpret_cast<const uint2 *>(mask + m * ldm + c);
            const __nv_bfloat16 *mh = reinterpret_cast<const __nv_bfloat16 *>(&mr);
#pragma unroll
            for (int j = 0; j < 4; ++j) v[j] = (__bfloat162float(mh[j]) > 0.f) ? v[j] : 0.f;
        }
        uint2 o;
        o.x = pack_bf16(v[0], v[1]);
        o.y = pack_bf16(v[2], v[3]);
        *reinterpret_cast<uint2 *>(out + m * ldo + c) = o;
    }
}

}  // namespace

bool tma_map_bf16(CUtensorMap *map, const void *base, long inner, long outer, long ld_elems, int box_inner,
                  int box_outer) {
    return make_map(map, base, inner, outer, ld_elems, box_inner, box_outer, false, 128);
}

// Split-K is used for the small-M GEMMs of a minibatch (forward X W^T and dX = G W at
// M = B = 256): with one output tile per SM they are L2->SM bandwidth bound because every
// N-tile re-reads the activations; fewer, wider (BN = 256) tiles cut that traffic and the
// K splits restore the parallelism.  Returns the split count (1 = not used).
static int env_int(const char *name, int dflt) {
    const char *v = getenv(name);
    return v ? atoi(v) : dflt;
}

// 2-CTA pairs (M = 256 per MMA) for every plain GEMM with at least 256 rows
static int use_pairs(const Gemm &g) {
    if (env_int("PD_GEMM_CG", 2) == 1) return 1;
    // N <= 64 would leave the second CTA's half of B empty (zero columns) with 128-wide pair
    // tiles -- except the implicit-GEMM conv forward at N = 64 (K-major weights), which runs
    // 256 x 64 pair tiles (each CTA stages 32 weight rows: 20 KB per K-block instead of 24)
    if (g.M >= 256 && g.N == 64 && g.conv.taps && g.bmaj == KMAJ && g.epi == EPI_STORE && !g.conv.c8) return 2;
    return (g.M >= 256 && g.N > 64 && (g.epi == EPI_STORE || g.epi == EPI_MASK || g.epi == EPI_F32)) ? 2 : 1;
}

// Cluster split-K (tc_gemm_csplit_kernel) for the small-M forward / dX GEMMs: the S K-splits
// of each 128 x 256 tile reduced through DSMEM.  S = the widest split in {4, 2} whose CTAs
// (tiles x S) fit the machine with >= 4 K-blocks per split; 0 = not applicable.
// PD_GEMM_CSPLIT=0 selects the workspace split-K path instead (tools / tests).
static int choose_csplit(const Gemm &g, int sms) {
    if (!(g.epi == EPI_STORE || g.epi == EPI_MASK) || g.conv.taps || g.amaj != KMAJ || g.N % 8 || g.M > 512)
        return 0;
    const int mode = env_int("PD_GEMM_CSPLIT", 2);
    if (mode == 0) return 0;
    const int kblocks = (g.K + BK - 1) / BK;
    if (mode == 2) {  // pairs, 2 K halves (tc_gemm_csplit2_kernel): returns -2
        const long ctas = (long)((g.M + 255) / 256) * ((g.N + 127) / 128) * 4;
        if (ctas <= sms && kblocks >= 8) return -2;
    }
    const long tiles = (long)((g.M + BM - 1) / BM) * ((g.N + 255) / 256);
    for (int S : {4, 2}) {
        const int kper = (kblocks + S - 1) / S;
        if (tiles * S <= sms && kper >= 4 && (S - 1) * kper < kblocks) return S;
    }
    return 0;
}

static int choose_ksplit(const Gemm &g, int sms) {
    if (!(g.epi == EPI_STORE || g.epi == EPI_MASK) || !g.workspace || g.N % 4 || g.ldo != g.N || g.conv.taps)
        return 1;
    const int forced = env_int("PD_GEMM_SPLIT", 0);  // tuning override (tools/gemm_bench.py)
    if (forced > 0) return forced;
    const int cg = use_pairs(g);
    const long slots = sms / cg;  // CTAs (or pairs) that can run at once
    const long tiles = (long)((g.M + BM * cg - 1) / (BM * cg)) * ((g.N + 255) / 256);
    const int kblocks = (g.K + BK - 1) / BK;
    if (tiles * 2 > slots) return 1;
    int S = (int)(slots / tiles);
    if (S > 8) S = 8;
    while (S > 1 && kblocks / S < 8) --S;
    while (S > 1 && (long)S * g.M * g.N * 4 > g.workspace_bytes) --S;
    const int kper = (kblocks + S - 1) / S;
    return (kblocks + kper - 1) / kper;  // no empty K range
}

// packed-tap convolution GEMMs for Cp = 8 inputs (ConvGeom::c8); single CTAs, BN = 128
// template (ring stages of 32 KB hold the 20 KB A + 10 KB B packed K-block)
static cudaError_t gemm_c8(const Gemm &g, cudaStream_t s) {
    CUtensorMap ma, mbm;
    EpiArgs e{};
    e.conv = g.conv;
    e.out = g.out;
    e.ldo = g.ldo;
    e.bias = g.bias;
    e.relu = g.relu;
    e.ksplit = 1;
    if (g.conv.c8 == 1 && g.lda == 8 && g.conv.Wp > 0) {
        // forward: one contiguous span of X rows per tile (conv_c8_fwd_kernel); W resident
        if (g.N > 64 || g.amaj != KMAJ || g.bmaj != KMAJ || g.epi != EPI_STORE) return cudaErrorInvalidValue;
        CUtensorMap mo;
        if (!make_map(&mbm, g.B, 72, g.N, g.ldb, 8, 64, false, 0) || !make_map(&mo, g.out, g.N, g.M, g.ldo, 32, 32, false, 64))
            return cudaErrorInvalidValue;
        const int span = ((BM + 2 * (g.conv.Wp + 1)) * 16 + 1023) / 1024 * 1024;
        const int smem = 10 * 1024 + C8_NS * span + 8 * 4096 + 256 + 1024;
        if (smem > 232448) return cudaErrorInvalidValue;
        static int attr_smem = 0;
        if (smem > attr_smem) {
            cudaError_t err = cudaFuncSetAttribute(conv_c8_fwd_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
            if (err != cudaSuccess) return err;
            attr_smem = smem;
        }
        const int tiles = (g.M + BM - 1) / BM;
        const int grid = tiles < num_sms() ? tiles : num_sms();
        conv_c8_fwd_kernel<<<grid, C8_THREADS, smem, s>>>(mbm, mo, static_cast<const __nv_bfloat16 *>(g.A), e, g.M, g.N,
                                                          span);
        ++tl_launches;
        return cudaGetLastError();
    }
    if (g.conv.c8 == 1) {
        // forward without the output grid (no halo geometry): A = X [M][8] (box {8, 128}),
        // B = W [N][72] (box {8, N}); N <= 64
        if (g.N > 64 || g.amaj != KMAJ || g.bmaj != KMAJ || g.epi != EPI_STORE) return cudaErrorInvalidValue;
        if (!make_map(&ma, g.A, 8, g.M, g.lda, 8, BM, false, 0) ||
            !make_map(&mbm, g.B, 72, g.N, g.ldb, 8, 64, false, 0))
            return cudaErrorInvalidValue;
        Gemm gg = g;
        gg.K = BK;  // one packed K-block per tile
        return dispatch_epi<128, KMAJ, KMAJ, 1>(gg, ma, mbm, e, s);
    }
    // weight gradient: A = dY [K pixels][M = Cout] MN-major, B = X [K pixels][8] shifted per tap
    if (g.N != 72 || g.amaj != MNMAJ || g.bmaj != MNMAJ || g.epi != EPI_F32 || !g.atomic_out)
        return cudaErrorInvalidValue;
    if (!make_map(&ma, g.A, g.M, g.K, g.lda, 64, BK) || !make_map(&mbm, g.B, 8, g.K, g.ldb, 8, BK, false, 0))
        return cudaErrorInvalidValue;
    e.atomic_out = 1;
    const int sms = num_sms();
    const long tiles = (g.M + BM - 1) / BM;
    const int kb = (g.K + BK - 1) / BK;
    long S = (2L * sms + tiles - 1) / tiles;  // (2, 4 and 8 units per SM measured equal here)
    if (S > kb / 4) S = kb / 4;
    if (S < 1) S = 1;
    const long kper = (kb + S - 1) / S;
    e.ksplit = (int)((kb + kper - 1) / kper);
    return dispatch_epi<128, MNMAJ, MNMAJ, 1>(g, ma, mbm, e, s);
}

cudaError_t gemm_bf16(const Gemm &g, cudaStream_t s) {
    if (g.M <= 0 || g.N <= 0 || g.K <= 0) return cudaErrorInvalidValue;
    if (const int S = choose_csplit(g, num_sms())) {
        CUtensorMap ma, mbm;
        const bool okA = make_map(&ma, g.A, g.K, g.M, g.lda, 64, BM);
        const bool okB = g.bmaj == KMAJ ? make_map(&mbm, g.B, g.K, g.N, g.ldb, 64, S < 0 ? 64 : 256)
                                        : make_map(&mbm, g.B, g.N, g.K, g.ldb, 64, BK);
        if (!okA || !okB) return cudaErrorInvalidValue;
        EpiArgs e{};
        e.out = g.out;
        e.ldo = g.ldo;
        e.ksplit = S;
        e.bias = g.bias;
        e.relu = g.relu;
        e.mask = static_cast<const __nv_bfloat16 *>(g.mask);
        e.ldm = g.ldm;
        if (S < 0) {
            if (g.bmaj == KMAJ) return g.epi == EPI_STORE ? launch_csplit2<KMAJ, KMAJ, EPI_STORE>(g, ma, mbm, e, s)
                                                          : launch_csplit2<KMAJ, KMAJ, EPI_MASK>(g, ma, mbm, e, s);
            return g.epi == EPI_STORE ? launch_csplit2<KMAJ, MNMAJ, EPI_STORE>(g, ma, mbm, e, s)
                                      : launch_csplit2<KMAJ, MNMAJ, EPI_MASK>(g, ma, mbm, e, s);
        }
        if (g.epi == EPI_STORE) return S == 4 ? csplit_major<EPI_STORE, 4>(g, ma, mbm, e, s) : csplit_major<EPI_STORE, 2>(g, ma, mbm, e, s);
        return S == 4 ? csplit_major<EPI_MASK, 4>(g, ma, mbm, e, s) : csplit_major<EPI_MASK, 2>(g, ma, mbm, e, s);
    }
    {
        const int S = choose_ksplit(g, num_sms());
        if (S > 1) {
            CUtensorMap ma, mbm;
            const int cg = use_pairs(g);
            const bool okA = g.amaj == KMAJ ? make_map(&ma, g.A, g.K, g.M, g.lda, 64, BM)
                                            : make_map(&ma, g.A, g.M, g.K, g.lda, 64, BK);
            const bool okB = g.bmaj == KMAJ ? make_map(&mbm, g.B, g.K, g.N, g.ldb, 64, 256 / cg)
                                            : make_map(&mbm, g.B, g.N, g.K, g.ldb, 64, BK);
            if (!okA || !okB) return cudaErrorInvalidValue;
            EpiArgs e{};
            e.conv = g.conv;
            e.out = g.workspace;
            e.ldo = g.N;
            e.ksplit = S;
            e.split_stride = (long)g.M * g.N;
            // zeroed workspace (kernel ABI workspace_zeroed): every split reduce-adds (TMA, in L2)
            // into one fp32 partial set, the reduction kernel reads M*N instead of S*M*N floats
            // and re-zeroes them
            const bool atomic = g.ws_zeroed;
            if (atomic) {
                e.atomic_out = 1;
                e.split_stride = 0;
            }
            Gemm gf = g;
            gf.epi = EPI_F32;
            cudaError_t err = cg == 2 ? dispatch_major<256, 2>(gf, ma, mbm, e, s) : dispatch_major<256>(gf, ma, mbm, e, s);
            if (err != cudaSuccess) return err;
            const long total = (long)g.M * (g.N / 4);
            long blocks = (total + 255) / 256;
            if (blocks > 148L * 8) blocks = 148L * 8;
            ++tl_launches;
            splitk_epilogue_kernel<<<(unsigned)blocks, 256, 0, s>>>(
                (const float *)g.workspace, atomic ? 1 : S, (long)g.M * g.N, g.M, g.N,
                g.epi == EPI_STORE ? g.bias : nullptr, g.epi == EPI_STORE ? g.relu : 0,
                g.epi == EPI_MASK ? static_cast<const __nv_bfloat16 *>(g.mask) : nullptr, g.ldm,
                static_cast<__nv_bfloat16 *>(g.out), g.ldo, atomic ? g.workspace : nullptr);
            return cudaGetLastError();
        }
    }
    if ((g.epi == EPI_SGD || g.epi == EPI_ADAM) && g.ldo == g.N && g.N % 8 == 0) return gemm_bf16_update(g, s);
    if (g.conv.c8) return gemm_c8(g, s);
    if (g.M <= 0 || g.N <= 0 || g.K <= 0) return cudaErrorInvalidValue;
    // tile width: the widest BN that still gives every SM a tile
    const int sms = num_sms();
    const int mb = (g.M + BM - 1) / BM;
    const int cg = use_pairs(g);
    int BN = 256;
    if (cg == 2) {
        // pair tiles of 256 rows; BN >= 128 so each CTA holds >= 64 B columns
        const long pm = (g.M + 255) / 256;
        // operand bytes each CTA ingests per K-block (32 KB at BN 256, 24 KB at BN 128) x
        // waves of pair tiles: the per-SM TMA ingest bounds these GEMMs (tools/tma_bw.cu)
        const long slots = sms / 2, t256 = pm * ((g.N + 255) / 256), t128 = pm * ((g.N + 127) / 128);
        const long c256 = (t256 + slots - 1) / slots * 32, c128 = (t128 + slots - 1) / slots * 24;
        if (c128 < c256 || g.N <= 128) BN = 128;
        if (g.N <= 64) BN = 64;  // (use_pairs allows it for the conv forward only)
    } else {
        if ((long)mb * ((g.N + 255) / 256) < sms || g.N <= 128) BN = 128;
        if (BN == 128 && ((long)mb * ((g.N + 127) / 128) < sms || g.N <= 64)) BN = 64;
    }
    // long-K reductions split K to fill the machine (atomic_out, ksplit 0: conv weight
    // gradients over N*H*W pixels), so narrow tiles buy no parallelism -- only ingest: the
    // widest tile has the most FLOPs per streamed byte (128 x 256 x 64 per 48 KB vs 128 x 64 x 64
    // per 24 KB; the ingest of ~90 GB/s per SM bounds these tiles)
    if (g.atomic_out && g.ksplit == 0 && g.N >= 256 && !g.conv.c8) BN = 256;
    BN = env_int("PD_GEMM_BN", BN);  // tuning override (tools/gemm_bench.py)
    if (cg == 2 && BN < 128 && g.N > 64) BN = 128;
    CUtensorMap ma, mbm;
    // implicit-GEMM conv: the tensors are [rows][channels] / [Cout][9*Cp]; the K walk over
    // (tap, channel block) is done by the producer's coordinates, not by the map extents
    const long aK = g.conv.taps ? g.conv.a_inner : g.K;
    const long bK = g.conv.taps && g.bmaj == KMAJ ? g.conv.b_inner : g.K;
    const long bN = g.conv.taps && g.bmaj == MNMAJ ? g.conv.b_inner : g.N;
    const long bKo = g.conv.taps && g.bmaj == MNMAJ ? g.conv.a_inner : g.K;  // dX: k = Cout rows of W
    const bool okA = g.amaj == KMAJ ? make_map(&ma, g.A, aK, g.M, g.lda, 64, BM)
                                    : make_map(&ma, g.A, g.M, g.K, g.lda, 64, BK);
    const bool okB = g.bmaj == KMAJ ? make_map(&mbm, g.B, bK, g.N, g.ldb, 64, BN / cg)
                                    : make_map(&mbm, g.B, g.conv.b_tapchunk ? g.conv.b_tapchunk : bN, bKo, g.ldb, 64, BK);
    if (!okA || !okB) return cudaErrorInvalidValue;
    EpiArgs e{};
    e.conv = g.conv;
    e.atomic_out = g.atomic_out;
    e.out = g.out;
    e.ldo = g.ldo;
    e.ksplit = g.ksplit > 1 ? g.ksplit : 1;
    if (g.atomic_out && g.ksplit == 0) {  // long-K reductions (conv dW): fill the machine
        const long tiles = (long)mb * ((g.N + BN - 1) / BN);
        const int kb = (g.K + BK - 1) / BK;
        // ~8 (tile, K-range) units per SM: shorter ranges balance the persistent CTAs and keep
        // the concurrently streamed pixel windows close together in L2 (measured on VGG-16: 2 ->
        // 4 -> 8 -> 16 -> 32 units per SM: 5.85k, 6.16k, 6.32k, 6.30k, 6.09k samples/s)
        long S = (8L * sms + tiles - 1) / tiles;
        if (S > kb / 4) S = kb / 4;
        if (S < 1) S = 1;
        const long kper = (kb + S - 1) / S;
        e.ksplit = (int)((kb + kper - 1) / kper);  // no empty K range
    }
    if (e.ksplit > 1) {
        const int kb = (g.K + BK - 1) / BK;
        const int kper = (kb + e.ksplit - 1) / e.ksplit;
        e.ksplit = (kb + kper - 1) / kper;
    }
    e.split_stride = 0;
    e.wait_cnt = g.wait_cnt;
    e.wait_T = g.wait_T;
    e.wait_B = g.wait_B > 0 ? g.wait_B : 1;
    e.wait_per = g.wait_per;
    if (g.wait_cnt && (g.epi != EPI_F32 || !g.atomic_out || g.conv.taps)) return cudaErrorInvalidValue;
    e.bias = g.bias;
    e.relu = g.relu;
    e.mask = static_cast<const __nv_bfloat16 *>(g.mask);
    e.ldm = g.ldm;
    e.master = g.master;
    e.slot = static_cast<__nv_bfloat16 *>(g.slot);
    e.adam_m = g.adam_m;
    e.adam_v = g.adam_v;
    e.lr = g.lr;
    e.b1 = g.b1;
    e.b2 = g.b2;
    e.eps = g.eps;
    e.bc1 = 1.f - powf(g.b1, (float)g.step);
    e.bc2 = 1.f - powf(g.b2, (float)g.step);
    if (cg == 2) {
        if (BN == 256) return dispatch_major<256, 2>(g, ma, mbm, e, s);
        if (BN == 64) return launch<64, KMAJ, KMAJ, EPI_STORE, 2>(g, ma, mbm, e, s);  // (use_pairs: conv fwd only)
        return dispatch_major<128, 2>(g, ma, mbm, e, s);
    }
    if (BN == 256) return dispatch_major<256>(g, ma, mbm, e, s);
    if (BN == 128) return dispatch_major<128>(g, ma, mbm, e, s);
    return dispatch_major<64>(g, ma, mbm, e, s);
}

}  // namespace pd
