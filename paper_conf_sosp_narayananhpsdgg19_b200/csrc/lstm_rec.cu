// lstm_rec.cu -- persistent, weight-stationary LSTM recurrences on the tcgen05 tensor cores.
//
// The recurrent half of an LSTM layer (R22, PyTorch form, gates i, f, g, o) is a
// chain of T small GEMMs (M = B = 64 rows, K = H) that the per-step path runs as T x (GEMM +
// cell kernel) launches.  Here ONE launch runs the whole chain:
//
//   * W_hh is split over the grid once and stays in shared memory (128B-swizzled K-major
//     UMMA tiles) for all T steps;
//   * each step's operand (h[t-1] forward, da[t+1] backward) is TMA-loaded straight from the
//     buffer the previous step wrote, as soon as the CTAs that produce its 64-column K-block
//     have published it (per-K-block counters: release-add by the producers, acquire-poll by
//     the consumer -- a dependency, not a grid-wide barrier);
//   * the cluster splits K: each CTA of a cluster multiplies its K-range into a TMEM partial
//     (M = 128 weight rows, N = batch), the partials are summed through distributed shared
//     memory in CTA-rank order (deterministic), and the cell (forward) or cell-backward is
//     applied by the CTA that owns the units, with c (forward) / dc (backward) kept in
//     registers across steps.
//
//   forward : cluster of 4 CTAs owns 32 hidden units = 128 gate rows (row = g*32 + unit);
//             CTA r multiplies K-range [r*H/4, (r+1)*H/4) of h[t-1]; owns 8 units.
//   backward: cluster of 8 CTAs owns 128 hidden units (row = unit); CTA r multiplies gate
//             rows [r*H/2, (r+1)*H/2) of da[t+1] against W_hh^T; owns 16 units.
//
// Semantics are those of lstm_cell_fwd/_bwd in lstm.cu + the recurrent GEMMs (bf16 operands,
// fp32 accumulation, bf16 h / da); only the fp32 summation order differs.
#include <cuda_bf16.h>

#include <cstdio>
#include <cstdlib>

#include "pd_internal.h"
#include "tc_ptx.h"

namespace pd {
namespace {
using namespace tcx;

constexpr int RT = 128;           // 4 warps = the 4 TMEM lane quadrants
constexpr int TILE_W = 128 * 128;  // one [128 rows][64 K] bf16 SW128 tile (bytes)
constexpr int TILE_X = 64 * 128;   // one [<=64 rows][64 K] bf16 SW128 tile (bytes)
constexpr int RECV_BYTES = 128 * 64 * 4;  // partials pushed to this CTA: [src][rows it owns][64 b]

__device__ __forceinline__ float sigm(float x) { return 1.0f / (1.0f + __expf(-x)); }

__device__ __forceinline__ unsigned ld_acquire(const unsigned *p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned long long gtime() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
// wait until *p >= target; a dependency that never arrives (a non-resident grid) traps after
// ~4 s instead of hanging the device
__device__ __forceinline__ void wait_count(const unsigned *p, unsigned target) {
    if (ld_acquire(p) >= target) return;
    const unsigned long long t0 = gtime();
    while (ld_acquire(p) < target) {
        if (gtime() - t0 > 4000000000ull) {
            printf("lstm_rec: dependency timeout (counter %u < %u)\n", ld_acquire(p), target);
            __trap();
        }
    }
}
__device__ __forceinline__ void fence_proxy_async_global() { asm volatile("fence.proxy.async.global;" ::: "memory"); }
// split cluster barrier: arrive after the DSMEM reads of a step, wait before this CTA next
// overwrites what its peers read (its staging buffer / the tiles the staging aliases)
__device__ __forceinline__ void cl_arrive() { asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory"); }
__device__ __forceinline__ void cl_sync() {
    asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory");
    asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ void cl_wait() { asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory"); }
__device__ __forceinline__ void st_dsmem_v4(uint32_t addr, float a, float b, float c, float d) {
    asm volatile("st.shared::cluster.v4.f32 [%0], {%1, %2, %3, %4};" ::"r"(addr), "f"(a), "f"(b), "f"(c), "f"(d)
                 : "memory");
}
__device__ __forceinline__ void red_relaxed_add(unsigned *p, unsigned v) {
    asm volatile("red.relaxed.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void fence_acq_rel_gpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
// publish one step: release-add (orders this CTA's earlier stores, seen through bar.sync)
__device__ __forceinline__ void red_release_add(unsigned *p, unsigned v) {
    asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
// byte offset of element (row, k) of a [rows][64] bf16 K-major tile, 128B swizzle
__device__ __forceinline__ uint32_t sw128(int row, int k) {
    return (uint32_t)((row >> 3) * 1024 + (row & 7) * 128 + ((((k >> 3) ^ row) & 7) << 4) + (k & 7) * 2);
}
__device__ __forceinline__ void tmem_alloc(uint32_t dst_smem, uint32_t cols) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(dst_smem), "r"(cols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
}
__device__ __forceinline__ void tmem_free(uint32_t taddr, uint32_t cols) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(cols));
}

struct RecArgs {
    int T, B, H, N;         // N = MMA N = roundup(B, 16)
    unsigned *cnt;          // per 64-column K-block counters
    const __nv_bfloat16 *W; // W_hh [4H][H]
    // forward
    const float *gx, *b_ih, *b_hh;
    float *gates, *c;
    __nv_bfloat16 *h;
    // backward
    const __nv_bfloat16 *dy;
    const float *gates_in, *c_in;
    __nv_bfloat16 *da;
    unsigned long long *probe;  // tools: [grid][T][8] %globaltimer stamps by thread 0 (nullptr = off)
};

__device__ __forceinline__ void stamp(const RecArgs &a, int step, int k) {
    if (a.probe && threadIdx.x == 0) a.probe[((long)blockIdx.x * a.T + step) * 8 + k] = gtime();
}

// After the MMAs of a step every CTA holds an fp32 partial D[128 rows][N] (TMEM lane = row).
// Thread `row` pushes its 64 batch columns into the receive buffer of the CTA that owns the
// row with st.async (16 x 16 B into distributed shared memory), each completing its bytes on
// the owner's receive mbarrier -- a point-to-point handoff, no cluster-wide barrier.
// dst_off = byte offset of this row's 64 floats in the owner's buffer.
__device__ __forceinline__ void push_partial(uint32_t tmem, int warp, uint32_t recv_s, uint32_t rbar, int owner,
                                             uint32_t dst_off) {
    const uint32_t base = mapa_cluster(recv_s + dst_off, owner);
    const uint32_t bar = mapa_cluster(rbar, owner);
#pragma unroll
    for (int ch = 0; ch < 2; ++ch) {
        float v[32];
        tmem_ld32(tmem + ((uint32_t)(warp * 32) << 16) + ch * 32, v);
#pragma unroll
        for (int q = 0; q < 8; ++q)
            asm volatile(
                "st.async.shared::cluster.mbarrier::complete_tx::bytes.v4.f32 [%0], {%1, %2, %3, %4}, [%5];" ::"r"(
                    base + (ch * 32 + q * 4) * 4),
                "f"(v[q * 4]), "f"(v[q * 4 + 1]), "f"(v[q * 4 + 2]), "f"(v[q * 4 + 3]), "r"(bar)
                : "memory");
    }
}

// MMA issue for one step: KB K-blocks of 64, D[128][N] (+)= A_kb[128][64] . B_kb[N][64]^T
// A_kb is K-major ([128 rows][64 K], forward) or MN-major (two [64 K][64 rows] chunks 8 KB
// apart, backward: W_hh tiles loaded untransposed)
template <int AMN>
__device__ __forceinline__ void issue_mmas(uint32_t tmem, uint32_t a_base, uint32_t b_base, uint32_t full0,
                                           uint32_t mma_bar, int KB, int N, uint32_t parity) {
    const uint32_t idesc = make_idesc(128, N, AMN, 0);
    for (int kb = 0; kb < KB; ++kb) {
        mbar_wait(full0 + kb * 8, parity);
        tc_fence_after();
#pragma unroll
        for (int kk = 0; kk < 4; ++kk) {
            const uint64_t ad = AMN ? smem_desc(a_base + kb * TILE_W + kk * 2048, 8192, 1024)
                                    : smem_desc(a_base + kb * TILE_W + kk * 32, 16, 1024);
            const uint64_t bd = smem_desc(b_base + kb * TILE_X + kk * 32, 16, 1024);
            tc_mma(tmem, ad, bd, idesc, (kb | kk) != 0);
        }
    }
    tc_commit(mma_bar);
}

// ------------------------------------------------------------------------------ forward
__global__ void __launch_bounds__(RT, 1)
    lstm_rec_fwd_kernel(const __grid_constant__ CUtensorMap tmH, const __grid_constant__ CUtensorMap tmW, RecArgs a) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *sm = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    const int H = a.H, B = a.B, T = a.T, N = a.N;
    const int KB = H / 4 / 64;  // K-blocks per CTA
    uint8_t *sW = sm;                       // KB x [128][64] weight tiles
    uint8_t *sX = sW + KB * TILE_W;         // KB x [N][64] h tiles
    float *recv = reinterpret_cast<float *>(sX + KB * TILE_X);  // [src 4][g 4][u 8][b 64]
    uint64_t *bars = reinterpret_cast<uint64_t *>(reinterpret_cast<uint8_t *>(recv) + RECV_BYTES);
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(bars + 16);
    const uint32_t full0 = smem_u32(bars), mma_bar = smem_u32(bars + 8);

    const unsigned long long t_entry = gtime();
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int cr = (int)cluster_rank();
    const int cid = blockIdx.x / 4;
    const int U0c = cid * 32;           // cluster's first unit
    const int U0 = U0c + 8 * cr;        // this CTA's 8 units
    const int k0 = cr * (H / 4);        // this CTA's K-range of h

    // weights by TMA: tile kb rows g*32 .. g*32+31 <- W_hh[g*H + U0c .. +32][k0 + kb*64 .. +64]
    const uint32_t wbar = smem_u32(bars + 9), rbar = smem_u32(bars + 10);
    if (tid == 0) {
        for (int kb = 0; kb < KB; ++kb) mbar_init(full0 + kb * 8, 1);
        mbar_init(mma_bar, 1);
        mbar_init(wbar, 1);
        mbar_init(rbar, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        mbar_expect_tx(wbar, (uint32_t)KB * TILE_W);
        for (int kb = 0; kb < KB; ++kb)
            for (int g = 0; g < 4; ++g)
                tma_load_2d(smem_u32(sW + kb * TILE_W + g * 4096), &tmW, wbar, k0 + kb * 64, g * H + U0c);
    }
    if (warp == 0) tmem_alloc(smem_u32(tmem_slot), 64);
    fence_proxy_async();
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *tmem_slot;
    cluster_sync_all();  // every peer's receive mbarrier is initialised before the first push
    mbar_wait(wbar, 0);
    if (a.probe && tid == 0) {
        a.probe[(long)blockIdx.x * a.T * 8 + 6] = t_entry;
        a.probe[(long)blockIdx.x * a.T * 8 + 7] = gtime();
    }

    // finalize role: batch row b, units U0 + u4 .. +3
    const int b = tid & 63, u4 = (tid >> 6) * 4;
    const int j = U0 + u4;
    const bool act = b < B;
    float bs[4][4], cst[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
    for (int g = 0; g < 4; ++g) {
        const float4 x = *reinterpret_cast<const float4 *>(a.b_ih + g * H + j);
        const float4 y = *reinterpret_cast<const float4 *>(a.b_hh + g * H + j);
        bs[g][0] = x.x + y.x;
        bs[g][1] = x.y + y.y;
        bs[g][2] = x.z + y.z;
        bs[g][3] = x.w + y.w;
    }
    const uint32_t recv_s = smem_u32(recv);
    // push role: partial row m = warp*32 + lane = gate `warp`, cluster unit `lane` -> owner lane/8
    const uint32_t push_off = (uint32_t)(((cr * 4 + warp) * 8 + (lane & 7)) * 64 * 4);

    for (int t = 0; t < T; ++t) {
        stamp(a, t, 0);
        float gxv[4][4];
        if (act) {
#pragma unroll
            for (int g = 0; g < 4; ++g) {
                const float4 x = *reinterpret_cast<const float4 *>(a.gx + ((long)t * B + b) * 4 * H + g * H + j);
                gxv[g][0] = x.x;
                gxv[g][1] = x.y;
                gxv[g][2] = x.z;
                gxv[g][3] = x.w;
            }
        }
        float acc[4][4] = {};
        if (t > 0) {
            const uint32_t par = (uint32_t)(t - 1) & 1;
            if (t > 1) cl_wait();  // every owner finished reading the previous step's partials
            if (tid == 0) {
                // 64 units of h = 8 producer CTAs per K-block
                for (int kb = 0; kb < KB; ++kb) wait_count(a.cnt + (k0 >> 6) + kb, 8u * t);
                fence_proxy_async_global();
                for (int kb = 0; kb < KB; ++kb) {
                    mbar_expect_tx(full0 + kb * 8, (uint32_t)N * 128);
                    tma_load_2d(smem_u32(sX + kb * TILE_X), &tmH, full0 + kb * 8, k0 + kb * 64, (t - 1) * B);
                }
                stamp(a, t, 1);
            } else if (tid == 32) {
                issue_mmas<0>(tmem, smem_u32(sW), smem_u32(sX), full0, mma_bar, KB, N, par);
            }
            __syncwarp();
            mbar_wait(mma_bar, par);
            stamp(a, t, 2);
            tc_fence_after();
            if (tid == 0) mbar_expect_tx(rbar, 4u * 32 * 64 * 4);  // 4 sources x 32 rows x 64 b
            push_partial(tmem, warp, recv_s, rbar, lane >> 3, push_off);
            tc_fence_before();
            mbar_wait(rbar, par);
            stamp(a, t, 3);
            if (act) {
#pragma unroll
                for (int src = 0; src < 4; ++src)
#pragma unroll
                    for (int g = 0; g < 4; ++g)
#pragma unroll
                        for (int u = 0; u < 4; ++u) acc[g][u] += recv[((src * 4 + g) * 8 + u4 + u) * 64 + b];
            }
            cl_arrive();
            stamp(a, t, 4);
        }
        float ig[4], fg[4], gg[4], og[4], cc[4], hh[4];
        if (act) {
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                ig[u] = sigm(acc[0][u] + gxv[0][u] + bs[0][u]);
                fg[u] = sigm(acc[1][u] + gxv[1][u] + bs[1][u]);
                gg[u] = tanhf(acc[2][u] + gxv[2][u] + bs[2][u]);
                og[u] = sigm(acc[3][u] + gxv[3][u] + bs[3][u]);
                cc[u] = fg[u] * cst[u] + ig[u] * gg[u];
                hh[u] = og[u] * tanhf(cc[u]);
                cst[u] = cc[u];
            }
            // h first: it is what the next step waits for
            const long r1 = ((long)t * B + b) * H + j;
            uint2 p;
            p.x = pack_bf16(hh[0], hh[1]);
            p.y = pack_bf16(hh[2], hh[3]);
            *reinterpret_cast<uint2 *>(a.h + r1) = p;
        }
        __syncthreads();
        if (tid == 0 && t + 1 < T) {
            red_release_add(a.cnt + (U0 >> 6), 1u);
        }
        if (act) {
            const long r4 = ((long)t * B + b) * 4 * H + j;
            *reinterpret_cast<float4 *>(a.gates + r4) = make_float4(ig[0], ig[1], ig[2], ig[3]);
            *reinterpret_cast<float4 *>(a.gates + r4 + H) = make_float4(fg[0], fg[1], fg[2], fg[3]);
            *reinterpret_cast<float4 *>(a.gates + r4 + 2 * H) = make_float4(gg[0], gg[1], gg[2], gg[3]);
            *reinterpret_cast<float4 *>(a.gates + r4 + 3 * H) = make_float4(og[0], og[1], og[2], og[3]);
            *reinterpret_cast<float4 *>(a.c + ((long)t * B + b) * H + j) = make_float4(cc[0], cc[1], cc[2], cc[3]);
        }
        stamp(a, t, 5);
    }
    tc_fence_before();
    if (T > 1) cl_wait();  // no peer may push into / read from an exited CTA
    if (warp == 0) tmem_free(tmem, 64);
}

// ------------------------------------------------------------------------------ backward
__global__ void __launch_bounds__(RT, 1)
    lstm_rec_bwd_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmW, RecArgs a) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *sm = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    const int H = a.H, B = a.B, T = a.T, N = a.N;
    const int KB = H / 2 / 64;  // K-blocks of da per CTA
    uint8_t *sW = sm;                  // KB x [128 units][64 gate rows] = W_hh^T tiles
    uint8_t *sX = sW + KB * TILE_W;    // KB x [N][64] da tiles
    float *recv = reinterpret_cast<float *>(sX + KB * TILE_X);  // [src 8][u 16][b 64]
    uint64_t *bars = reinterpret_cast<uint64_t *>(reinterpret_cast<uint8_t *>(recv) + RECV_BYTES);
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(bars + 16);
    const uint32_t full0 = smem_u32(bars), mma_bar = smem_u32(bars + 8);

    const unsigned long long t_entry = gtime();
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int cr = (int)cluster_rank();
    const int cid = blockIdx.x / 8;
    const int U0c = cid * 128;       // cluster's first unit
    const int U0 = U0c + 16 * cr;    // this CTA's 16 units
    const int k0 = cr * (H / 2);     // this CTA's range of gate rows r

    // W_hh tiles by TMA, untransposed (MN-major A operand): tile kb = two [64 gate rows][64
    // units] chunks <- W_hh[k0 + kb*64 .. +64][U0c + 64 j .. +64]
    const uint32_t wbar = smem_u32(bars + 9), rbar = smem_u32(bars + 10);
    if (tid == 0) {
        for (int kb = 0; kb < KB; ++kb) mbar_init(full0 + kb * 8, 1);
        mbar_init(mma_bar, 1);
        mbar_init(wbar, 1);
        mbar_init(rbar, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        mbar_expect_tx(wbar, (uint32_t)KB * TILE_W);
        for (int kb = 0; kb < KB; ++kb)
            for (int jj = 0; jj < 2; ++jj)
                tma_load_2d(smem_u32(sW + kb * TILE_W + jj * 8192), &tmW, wbar, U0c + 64 * jj, k0 + kb * 64);
    }
    if (warp == 0) tmem_alloc(smem_u32(tmem_slot), 64);
    fence_proxy_async();
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *tmem_slot;
    cluster_sync_all();  // every peer's receive mbarrier is initialised before the first push
    mbar_wait(wbar, 0);
    if (a.probe && tid == 0) {
        a.probe[(long)blockIdx.x * a.T * 8 + 6] = t_entry;
        a.probe[(long)blockIdx.x * a.T * 8 + 7] = gtime();
    }

    // finalize role: batch row b, units U0 + u8 .. +7
    const int b = tid & 63, u8 = (tid >> 6) * 8;
    const int j = U0 + u8;
    const bool act = b < B;
    float dc[8] = {};
    const uint32_t recv_s = smem_u32(recv);
    // push role: partial row m = warp*32 + lane = cluster unit m -> owner m/16
    const int m = warp * 32 + lane;
    const uint32_t push_off = (uint32_t)((cr * 16 + (m & 15)) * 64 * 4);

    for (int s = 0; s < T; ++s) {
        const int t = T - 1 - s;
        stamp(a, s, 0);
        float dh[8], gi[8], gf[8], gg[8], go[8], ct[8], cp[8];
        if (act) {
            const long r1 = ((long)t * B + b) * H + j;
            const uint4 raw = *reinterpret_cast<const uint4 *>(a.dy + r1);
            const __nv_bfloat16 *hv = reinterpret_cast<const __nv_bfloat16 *>(&raw);
#pragma unroll
            for (int u = 0; u < 8; ++u) dh[u] = __bfloat162float(hv[u]);
            const long r4 = ((long)t * B + b) * 4 * H + j;
            float *dst[4] = {gi, gf, gg, go};
#pragma unroll
            for (int g = 0; g < 4; ++g) {
                const float4 x0 = *reinterpret_cast<const float4 *>(a.gates_in + r4 + g * H);
                const float4 x1 = *reinterpret_cast<const float4 *>(a.gates_in + r4 + g * H + 4);
                dst[g][0] = x0.x, dst[g][1] = x0.y, dst[g][2] = x0.z, dst[g][3] = x0.w;
                dst[g][4] = x1.x, dst[g][5] = x1.y, dst[g][6] = x1.z, dst[g][7] = x1.w;
            }
            const float4 c0 = *reinterpret_cast<const float4 *>(a.c_in + r1);
            const float4 c1 = *reinterpret_cast<const float4 *>(a.c_in + r1 + 4);
            ct[0] = c0.x, ct[1] = c0.y, ct[2] = c0.z, ct[3] = c0.w, ct[4] = c1.x, ct[5] = c1.y, ct[6] = c1.z,
            ct[7] = c1.w;
            if (t > 0) {
                const float4 p0 = *reinterpret_cast<const float4 *>(a.c_in + r1 - (long)B * H);
                const float4 p1 = *reinterpret_cast<const float4 *>(a.c_in + r1 - (long)B * H + 4);
                cp[0] = p0.x, cp[1] = p0.y, cp[2] = p0.z, cp[3] = p0.w, cp[4] = p1.x, cp[5] = p1.y, cp[6] = p1.z,
                cp[7] = p1.w;
            } else {
#pragma unroll
                for (int u = 0; u < 8; ++u) cp[u] = 0.f;
            }
        }
        if (s > 0) {
            const uint32_t par = (uint32_t)(s - 1) & 1;
            if (s > 1) cl_wait();  // every owner finished reading the previous step's partials
            if (tid == 0) {
                // 64 gate rows of da = 4 producer CTAs per K-block
                for (int kb = 0; kb < KB; ++kb) wait_count(a.cnt + (k0 >> 6) + kb, 4u * s);
                fence_proxy_async_global();
                for (int kb = 0; kb < KB; ++kb) {
                    mbar_expect_tx(full0 + kb * 8, (uint32_t)N * 128);
                    tma_load_2d(smem_u32(sX + kb * TILE_X), &tmA, full0 + kb * 8, k0 + kb * 64, (t + 1) * B);
                }
                stamp(a, s, 1);
            } else if (tid == 32) {
                issue_mmas<1>(tmem, smem_u32(sW), smem_u32(sX), full0, mma_bar, KB, N, par);
            }
            __syncwarp();
            mbar_wait(mma_bar, par);
            stamp(a, s, 2);
            tc_fence_after();
            if (tid == 0) mbar_expect_tx(rbar, 8u * 16 * 64 * 4);  // 8 sources x 16 rows x 64 b
            push_partial(tmem, warp, recv_s, rbar, m >> 4, push_off);
            tc_fence_before();
            mbar_wait(rbar, par);
            stamp(a, s, 3);
            if (act) {
                float rec[8] = {};
#pragma unroll
                for (int src = 0; src < 8; ++src)
#pragma unroll
                    for (int u = 0; u < 8; ++u) rec[u] += recv[((src * 16 + u8 + u) * 64) + b];
#pragma unroll
                for (int u = 0; u < 8; ++u) dh[u] += rec[u];
            }
            cl_arrive();
            stamp(a, s, 4);
        }
        if (act) {
            float di[8], df[8], dg[8], dog[8];
#pragma unroll
            for (int u = 0; u < 8; ++u) {
                const float tc = tanhf(ct[u]);
                dog[u] = dh[u] * tc * go[u] * (1.f - go[u]);
                const float dct = dh[u] * go[u] * (1.f - tc * tc) + dc[u];
                di[u] = dct * gg[u] * gi[u] * (1.f - gi[u]);
                df[u] = dct * cp[u] * gf[u] * (1.f - gf[u]);
                dg[u] = dct * gi[u] * (1.f - gg[u] * gg[u]);
                dc[u] = dct * gf[u];
            }
            const long r4 = ((long)t * B + b) * 4 * H + j;
            const float *src4[4] = {di, df, dg, dog};
#pragma unroll
            for (int g = 0; g < 4; ++g) {
                uint4 p;
                p.x = pack_bf16(src4[g][0], src4[g][1]);
                p.y = pack_bf16(src4[g][2], src4[g][3]);
                p.z = pack_bf16(src4[g][4], src4[g][5]);
                p.w = pack_bf16(src4[g][6], src4[g][7]);
                *reinterpret_cast<uint4 *>(a.da + r4 + g * H) = p;
            }
        }
        __syncthreads();
        if (tid == 0 && s + 1 < T) {
            fence_acq_rel_gpu();
#pragma unroll
            for (int g = 0; g < 4; ++g) red_relaxed_add(a.cnt + ((g * H + U0) >> 6), 1u);
        }
        stamp(a, s, 5);
    }
    tc_fence_before();
    if (T > 1) cl_wait();
    if (warp == 0) tmem_free(tmem, 64);
}

int fwd_smem(int H) { return (H / 256) * (TILE_W + TILE_X) + RECV_BYTES + 256 + 1024; }
int bwd_smem(int H) { return (H / 128) * (TILE_W + TILE_X) + RECV_BYTES + 256 + 1024; }

template <typename K>
cudaError_t launch_clustered(K kern, int grid, int csize, int smem, const CUtensorMap &map, const CUtensorMap &wmap,
                             const RecArgs &a, cudaStream_t s) {
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(RT);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = csize;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kern, map, wmap, a);
}

// can `grid` CTAs in clusters of `csize` (smem bytes each) all be resident at once?
// (the attribute is set to the largest size any supported H launches with, so launches of
// different H, from several host threads, never race on it)
bool coresident(const void *kern, int grid, int csize, int smem, int smem_max) {
    if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_max) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(RT);
    cfg.dynamicSmemBytes = smem;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = csize;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    int n = 0;
    if (cudaOccupancyMaxActiveClusters(&n, kern, &cfg) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return n * csize >= grid;
}

}  // namespace

bool lstm_rec_supported(int B, int H) {
    if (B < 1 || B > 64 || H < 256 || H > 1024 || H % 256) return false;
    static int cache[5] = {};  // per H / 256
    int &c = cache[H / 256];
    if (!c) {
        const bool ok = coresident((const void *)lstm_rec_fwd_kernel, H / 8, 4, fwd_smem(H), fwd_smem(1024)) &&
                        coresident((const void *)lstm_rec_bwd_kernel, H / 16, 8, bwd_smem(H), bwd_smem(1024));
        c = ok ? 1 : -1;
    }
    return c > 0;
}

cudaError_t lstm_rec_fwd(const float *gx, const float *b_ih, const float *b_hh, const __nv_bfloat16 *Whh,
                         float *gates, float *c, __nv_bfloat16 *h, unsigned *cnt, int T, int B, int H,
                         cudaStream_t s, unsigned long long *probe) {
    if (!lstm_rec_supported(B, H)) return cudaErrorNotSupported;
    RecArgs a{};
    a.T = T, a.B = B, a.H = H, a.N = (B + 15) / 16 * 16;
    a.cnt = cnt, a.W = Whh, a.gx = gx, a.b_ih = b_ih, a.b_hh = b_hh, a.gates = gates, a.c = c, a.h = h;
    a.probe = probe;
    CUtensorMap map;
    CUtensorMap wmap;
    if (!tma_map_bf16(&map, h, H, (long)T * B, H, 64, a.N) || !tma_map_bf16(&wmap, Whh, H, 4L * H, H, 64, 32))
        return cudaErrorInvalidValue;
    ++tl_launches;
    return launch_clustered(lstm_rec_fwd_kernel, H / 8, 4, fwd_smem(H), map, wmap, a, s);
}

cudaError_t lstm_rec_bwd(const __nv_bfloat16 *dy, const float *gates, const float *c, const __nv_bfloat16 *Whh,
                         __nv_bfloat16 *da, unsigned *cnt, int T, int B, int H, cudaStream_t s,
                         unsigned long long *probe) {
    if (!lstm_rec_supported(B, H)) return cudaErrorNotSupported;
    RecArgs a{};
    a.T = T, a.B = B, a.H = H, a.N = (B + 15) / 16 * 16;
    a.cnt = cnt, a.W = Whh, a.dy = dy, a.gates_in = gates, a.c_in = c, a.da = da;
    a.probe = probe;
    CUtensorMap map;
    CUtensorMap wmap;
    if (!tma_map_bf16(&map, da, 4L * H, (long)T * B, 4L * H, 64, a.N) || !tma_map_bf16(&wmap, Whh, H, 4L * H, H, 64, 64))
        return cudaErrorInvalidValue;
    ++tl_launches;
    return launch_clustered(lstm_rec_bwd_kernel, H / 16, 8, bwd_smem(H), map, wmap, a, s);
}

}  // namespace pd
