// lstm_wave.cu -- a stage's stack of LSTM layers as ONE wavefront kernel (bf16 path).
//
// Layer l's step t needs only layer l-1's step t (its input) and its own step t-1, so the
// L layers of a stage can run as a wavefront: at wave w every layer l with t = w - l in
// [0, T) advances one step, T + L - 1 waves instead of L * T dependent steps.  The per-step
// work is the gate GEMM with the input projection folded in,
//     forward   a[t] = [x_t | h_{t-1}] . [W_ih | W_hh]^T + b_ih + b_hh        (K = 2H)
//     backward dh[t] = dy[t] + da[t+1] W_hh + da^{l+1}[t] W_ih^{l+1}          (K = 8H)
// (dy of the stage's top layer comes from the stage's output gradient), which makes the
// recurrence a weight-streaming problem -- all L layers' weights pass through the SMs once
// per wave -- instead of a chain of latency-bound small GEMMs.
//
// Persistent, warp-specialised, one CTA per SM; every CTA owns a fixed list of work items
// (layer, tile of hidden units) and walks the waves in order:
//   warp 0  weight producer: TMA of the A tiles (weight rows) into an S-stage ring; runs ahead
//           of the dependencies (weights never wait);
//   warp 1  activation producer: waits for the item's inputs (per-layer step counters,
//           acquire) and TMAs the B tiles (x_t / h_{t-1} or da) into the same ring stages;
//   warp 2  MMA: tcgen05.mma M = 128, N = B rounded up to 16, into a double-buffered TMEM
//           accumulator;
//   warp 3  TMEM allocator;
//   warps 4-7 epilogue: the LSTM cell (forward) or cell backward, stores, then publish the
//           item (release) so dependent items of the next wave can start.
// forward tile = 32 units (128 gate rows, gate-major: row = g*32 + u, K-major weights);
// backward tile = 128 units (row = unit; W^T read untransposed as an MN-major operand).
// All dependencies point to an earlier wave, and every CTA processes its items in wave
// order, so the spin-waits cannot deadlock once the grid is resident.
#include <cuda_bf16.h>

#include <cstdio>
#include <algorithm>
#include <cstring>
#include <vector>

#include "pd_internal.h"
#include "tc_ptx.h"

namespace pd {
namespace {
using namespace tcx;

constexpr int NT = 256;
constexpr int ATILE = 128 * 128;         // [128 rows][64 K] bf16 (or 2 x [64 K][64 rows] MN-major)
constexpr int BTILE = 64 * 128;          // [<= 64 rows][64 K] bf16
constexpr int STAGE = ATILE + BTILE;
constexpr int STG_LD = 68;               // forward epilogue staging row stride (floats)
constexpr int STG_BYTES = 128 * STG_LD * 4;
constexpr int RECV_BYTES = 128 * 32 * 4;  // backward: the peer's partial for this CTA's batch half

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
__device__ __forceinline__ void wait_count(const unsigned *p, unsigned target) {
    if (ld_acquire(p) >= target) return;
    const unsigned long long t0 = gtime();
    while (ld_acquire(p) < target) {
        if (gtime() - t0 > 4000000000ull) {
            printf("lstm_wave: dependency timeout (counter %u < %u)\n", ld_acquire(p), target);
            __trap();
        }
    }
}
__device__ __forceinline__ void fence_proxy_async_global() { asm volatile("fence.proxy.async.global;" ::: "memory"); }
__device__ __forceinline__ float sigm(float x) { return 1.0f / (1.0f + __expf(-x)); }
template <int NE>
__device__ __forceinline__ void epi_sync_n() { asm volatile("bar.sync 1, %0;" ::"n"(NE) : "memory"); }

struct WaveLayer {
    const float *b_ih, *b_hh;  // forward
    float *gates, *c;          // saved state [T][B][4H], [T][B][H] (written fwd, read bwd)
    __nv_bfloat16 *h;          // forward output [T][B][H]
    __nv_bfloat16 *da;         // backward output [T][B][4H]
    float *dc;                 // backward carry [B][H] (scratch)
};

struct WaveMaps {
    CUtensorMap w_ih[LSTM_WAVE_MAX_L], w_hh[LSTM_WAVE_MAX_L];
    CUtensorMap act[LSTM_WAVE_MAX_L + 1];  // fwd: act[0] = stage input, act[l+1] = h of l; bwd: act[l] = da of l
};

struct WaveArgs {
    int L, T, B, H, N, tiles;  // tiles per layer
    WaveLayer layer[LSTM_WAVE_MAX_L];
    const __nv_bfloat16 *dy_top;  // backward: gradient w.r.t. the top layer's output [T][B][H]
    unsigned *cnt;                // per-layer completed (step, tile) items, zeroed by the caller
    unsigned long long *probe;    // tools only (PD_WAVE_PROBE): [CTA][visit < PROBE_V][8] %globaltimer
    int keep_layers;              // weights of layers < keep_layers load with L2 evict_last, the rest
                                  // evict_first (0: no hint): a fixed subset stays L2-resident across
                                  // waves instead of the whole run thrashing the 126 MB L2
};
constexpr int PROBE_V = 256;
// probe events per item visit: 0 weight producer first K-block issued, 1 activation producer
// dependencies satisfied, 2 MMA last K-block issued, 3 epilogue accumulator ready, 4 epilogue
// partials exchanged / staged, 6 thread 0's cell loop done, 7 all epilogue threads done,
// 5 epilogue item published (after the release fence)
__device__ __forceinline__ void probe(const WaveArgs &a, int v, int ev) {
    if (a.probe && v < PROBE_V) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        a.probe[((long)blockIdx.x * PROBE_V + v) * 8 + ev] = t;
    }
}

// the item sequence of this CTA (pair): items i = c + k * C (c = cluster index, C = clusters,
// i = l * tiles + tile), visited wave by wave; returns false when done
template <int CL>
struct ItemIter {
    int wave = 0, k = -1;
    __device__ bool next(const WaveArgs &a, bool bwd, int &l, int &tile, int &t) {
        const int items = a.L * a.tiles, waves = a.T + a.L - 1;
        while (wave < waves) {
            ++k;
            const int i = (int)(blockIdx.x / CL) + k * (int)(gridDim.x / CL);
            if (i >= items) {
                k = -1;
                ++wave;
                continue;
            }
            l = i / a.tiles;
            tile = i % a.tiles;
            t = bwd ? a.T - 1 - (wave - (a.L - 1 - l)) : wave - l;
            if (t >= 0 && t < a.T) return true;
        }
        return false;
    }
};

// K-blocks of an item: forward [x part (H/64) | h part (t > 0 ? H/64 : 0)];
// backward [da[t+1] part (t < T-1 ? 4H/64 : 0) | da^{l+1}[t] part (l < L-1 ? 4H/64 : 0)]
// The CTAs of a cluster split an item's K-blocks: this CTA (rank of csize) takes the global
// K-block indices [lo, hi); index kb < n0 is part 0, else part 1 (kb - n0).
struct ItemK {
    int n0, n1, lo, hi;
};
__device__ __forceinline__ ItemK item_k(const WaveArgs &a, bool bwd, int l, int t, int rank, int csize) {
    ItemK r;
    if (!bwd) {
        r.n0 = a.H / 64;
        r.n1 = t > 0 ? a.H / 64 : 0;
    } else {
        r.n0 = t < a.T - 1 ? 4 * a.H / 64 : 0;
        r.n1 = l < a.L - 1 ? 4 * a.H / 64 : 0;
    }
    const int tot = r.n0 + r.n1;
    r.lo = tot * rank / csize;
    r.hi = tot * (rank + 1) / csize;
    return r;
}
__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}

// 8 epilogue warps, two per TMEM lane quadrant: backward -- 16 batch rows each (the cell
// backward is the latency-bound part of a wave); forward -- one 32-column accumulator chunk
// each to stage, 8 of a thread's 16 units each in the cell
template <bool BWD>
__host__ __device__ constexpr int wave_threads() { return 384; }

template <bool BWD>
__global__ void __launch_bounds__(wave_threads<BWD>(), 1) lstm_wave_kernel(const __grid_constant__ WaveMaps m, const WaveArgs a) {
    constexpr int NE = wave_threads<BWD>() - 128;  // epilogue threads
    auto epi_sync = [] { epi_sync_n<NE>(); };
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *sm = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    // backward: a cluster of 2 CTAs splits every item's K-blocks; each finishes half the batch
    constexpr int S = BWD ? 8 : 7, CL = BWD ? 2 : 1;
    float *stg = reinterpret_cast<float *>(sm + S * STAGE);  // fwd staging / bwd receive buffer
    uint64_t *bars = reinterpret_cast<uint64_t *>(sm + S * STAGE + (BWD ? RECV_BYTES : STG_BYTES));
    // bars: full_w[S], full_x[S], empty[S], acc_full[2], acc_empty[2], recv_full, recv_empty
    const uint32_t fw0 = smem_u32(bars), fx0 = smem_u32(bars + S), em0 = smem_u32(bars + 2 * S);
    const uint32_t af0 = smem_u32(bars + 3 * S), ae0 = smem_u32(bars + 3 * S + 2);
    const uint32_t rfull = smem_u32(bars + 3 * S + 4), rempty = smem_u32(bars + 3 * S + 5);
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(bars + 3 * S + 6);
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int H = a.H, B = a.B, N = a.N;
    const int rank = BWD ? (int)cluster_rank() : 0;

    if (tid == 0) {
        for (int s = 0; s < S; ++s) {
            mbar_init(fw0 + 8 * s, 1);
            mbar_init(fx0 + 8 * s, 1);
            mbar_init(em0 + 8 * s, 1);
        }
        for (int b = 0; b < 2; ++b) {
            mbar_init(af0 + 8 * b, 1);
            mbar_init(ae0 + 8 * b, NE);
        }
        mbar_init(rfull, 1);
        mbar_init(rempty, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 3) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 128;" ::"r"(smem_u32(tmem_slot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    tc_fence_before();
    __syncthreads();
    if (BWD) cluster_sync_all();  // the peer's barriers exist before any remote arrive / st.async
    tc_fence_after();
    const uint32_t tmem = *tmem_slot;
    // published (step, tile, CTA) items of a layer per completed step
    const unsigned per_step = (unsigned)a.tiles * CL;

    if (warp == 0 && lane == 0) {
        // ---------------- weight producer
        ItemIter<CL> it;
        int l, tile, t, s = 0, pv = 0;
        uint32_t ph = 0;
        const uint64_t pol_last = l2_policy_evict_last(), pol_first = l2_policy_evict_first();
        while (it.next(a, BWD, l, tile, t)) {
            const ItemK ik = item_k(a, BWD, l, t, rank, CL);
            for (int kb = ik.lo; kb < ik.hi; ++kb) {
                mbar_wait(em0 + 8 * s, ph ^ 1);
                if (kb == ik.lo) probe(a, pv, 0);
                const uint32_t dst = smem_u32(sm + s * STAGE);
                mbar_expect_tx(fw0 + 8 * s, ATILE);
                const bool p1 = kb >= ik.n0;
                const int k = (p1 ? kb - ik.n0 : kb) * 64;
                // the layer whose weights this K-block reads
                const int lw = BWD && p1 ? l + 1 : l;
                const uint64_t pol = lw < a.keep_layers ? pol_last : pol_first;
                if (!BWD) {
                    const CUtensorMap *w = p1 ? &m.w_hh[l] : &m.w_ih[l];
                    for (int g = 0; g < 4; ++g) {
                        if (a.keep_layers) tma_load_2d_hint(dst + g * 4096, w, fw0 + 8 * s, k, g * H + tile * 32, pol);
                        else tma_load_2d(dst + g * 4096, w, fw0 + 8 * s, k, g * H + tile * 32);
                    }
                } else {
                    const CUtensorMap *w = p1 ? &m.w_ih[l + 1] : &m.w_hh[l];
                    for (int jj = 0; jj < 2; ++jj) {
                        if (a.keep_layers) tma_load_2d_hint(dst + jj * 8192, w, fw0 + 8 * s, tile * 128 + 64 * jj, k, pol);
                        else tma_load_2d(dst + jj * 8192, w, fw0 + 8 * s, tile * 128 + 64 * jj, k);
                    }
                }
                if (++s == S) s = 0, ph ^= 1;
            }
            ++pv;
        }
    } else if (warp == 1 && lane == 0) {
        // ---------------- activation producer (waits for the item's inputs)
        ItemIter<CL> it;
        int l, tile, t, s = 0, pv = -1;
        uint32_t ph = 0;
        while (it.next(a, BWD, l, tile, t)) {
            const ItemK ik = item_k(a, BWD, l, t, rank, CL);
            ++pv;
            if (ik.lo == ik.hi) continue;
            const bool need0 = ik.lo < ik.n0, need1 = ik.hi > ik.n0;
            if (!BWD) {
                if (l > 0) wait_count(a.cnt + l - 1, (unsigned)(t + 1) * per_step);  // x_t = h^{l-1}[t]
                if (need1) wait_count(a.cnt + l, (unsigned)t * per_step);            // h^l[t-1]
            } else {
                if (need0) wait_count(a.cnt + l, (unsigned)(a.T - 1 - t) * per_step);  // da^l[t+1]
                if (need1) wait_count(a.cnt + l + 1, (unsigned)(a.T - t) * per_step);  // da^{l+1}[t]
            }
            fence_proxy_async_global();
            probe(a, pv, 1);
            for (int kb = ik.lo; kb < ik.hi; ++kb) {
                mbar_wait(em0 + 8 * s, ph ^ 1);
                const uint32_t dst = smem_u32(sm + s * STAGE + ATILE);
                mbar_expect_tx(fx0 + 8 * s, (uint32_t)N * 128);
                const bool p1 = kb >= ik.n0;
                const int k = (p1 ? kb - ik.n0 : kb) * 64;
                if (!BWD) {
                    if (!p1) tma_load_2d(dst, &m.act[l], fx0 + 8 * s, k, t * B);
                    else tma_load_2d(dst, &m.act[l + 1], fx0 + 8 * s, k, (t - 1) * B);
                } else {
                    if (!p1) tma_load_2d(dst, &m.act[l], fx0 + 8 * s, k, (t + 1) * B);
                    else tma_load_2d(dst, &m.act[l + 1], fx0 + 8 * s, k, t * B);
                }
                if (++s == S) s = 0, ph ^= 1;
            }
        }
    } else if (warp == 2 && lane == 0) {
        // ---------------- MMA issuer
        const uint32_t idesc = make_idesc(128, N, BWD ? 1 : 0, 0);
        ItemIter<CL> it;
        int l, tile, t, s = 0, acc = 0, pv = 0;
        uint32_t ph = 0, aph[2] = {0, 0};
        while (it.next(a, BWD, l, tile, t)) {
            const ItemK ik = item_k(a, BWD, l, t, rank, CL);
            mbar_wait(ae0 + 8 * acc, aph[acc] ^ 1);  // epilogue drained this accumulator
            tc_fence_after();
            const uint32_t d = tmem + acc * 64;
            for (int kb = ik.lo; kb < ik.hi; ++kb) {
                mbar_wait(fw0 + 8 * s, ph);
                mbar_wait(fx0 + 8 * s, ph);
                tc_fence_after();
                const uint32_t sa = smem_u32(sm + s * STAGE), sb = sa + ATILE;
#pragma unroll
                for (int kk = 0; kk < 4; ++kk) {
                    const uint64_t ad = BWD ? smem_desc(sa + kk * 2048, 8192, 1024) : smem_desc(sa + kk * 32, 16, 1024);
                    const uint64_t bd = smem_desc(sb + kk * 32, 16, 1024);
                    tc_mma(d, ad, bd, idesc, (kb > ik.lo || kk) ? 1u : 0u);
                }
                tc_commit(em0 + 8 * s);
                if (++s == S) s = 0, ph ^= 1;
            }
            probe(a, pv++, 2);
            if (ik.hi > ik.lo) tc_commit(af0 + 8 * acc);
            else mbar_arrive(af0 + 8 * acc);  // nothing to multiply: the epilogue uses 0
            aph[acc] ^= 1;
            acc ^= 1;
        }
    } else if (warp >= 4) {
        // ---------------- epilogue
        const int q = (warp - 4) & 3;   // TMEM lane quadrant (warp % 4)
        const int half = (warp - 4) >> 2;  // backward: which 16 of the 32 batch rows
        const int et = tid - 128;
        ItemIter<CL> it;
        int l, tile, t, acc = 0, pv = 0;
        uint32_t aph[2] = {0, 0}, rph = 0, eph = 0;
        while (it.next(a, BWD, l, tile, t)) {
            const ItemK ik = item_k(a, BWD, l, t, rank, CL);
            const bool mm = ik.hi > ik.lo;
            if (BWD) {
                // while the MMA runs: pull this item's cell-backward inputs (saved gates, c[t],
                // c[t-1], the dc carry; written long before, mostly in HBM) into L2 -- lane i of
                // warp q fetches the 128-byte lines of batch row hb + i for units q*32 .. q*32+31
                const int b = rank * 32 + lane, jq = tile * 128 + q * 32;
                if (half == 0 && b < B) {
                    const WaveLayer &Lp = a.layer[l];
                    const long r1 = ((long)t * B + b) * H + jq, r4 = ((long)t * B + b) * 4 * H + jq;
#pragma unroll
                    for (int g = 0; g < 4; ++g)
                        asm volatile("prefetch.global.L2 [%0];" ::"l"(Lp.gates + r4 + (long)g * H));
                    asm volatile("prefetch.global.L2 [%0];" ::"l"(Lp.c + r1));
                    if (t > 0) asm volatile("prefetch.global.L2 [%0];" ::"l"(Lp.c + r1 - (long)B * H));
                    if (t < a.T - 1) asm volatile("prefetch.global.L2 [%0];" ::"l"(Lp.dc + (long)b * H + jq));
                }
            }
            mbar_wait(af0 + 8 * acc, aph[acc]);
            aph[acc] ^= 1;
            tc_fence_after();
            if (et == 0) probe(a, pv, 3);
            const uint32_t d = tmem + acc * 64 + ((uint32_t)(q * 32) << 16);
            const WaveLayer &Ly = a.layer[l];
            if (!BWD) {
                // stage D[row = g*32 + u][b] so one thread sees all four gates of (u, b)
                const int row = q * 32 + lane;
                constexpr int NWQ = NE / 128;  // epilogue warps per TMEM lane quadrant
#pragma unroll
                for (int ch = half; ch < 2; ch += NWQ) {
                    float v[32];
                    tmem_ld32(d + ch * 32, v);
#pragma unroll
                    for (int i = 0; i < 8; ++i)
                        *reinterpret_cast<float4 *>(stg + row * STG_LD + ch * 32 + i * 4) =
                            make_float4(v[i * 4], v[i * 4 + 1], v[i * 4 + 2], v[i * 4 + 3]);
                }
                // gate row `row` = g*32 + u: b_ih + b_hh into the staging row's spare column 64
                // (STG_LD = 68), so the cell loop below reads biases from shared memory
                if (half == 0) {
                    const int gi = row >> 5, uu = row & 31, jb = gi * H + tile * 32 + uu;
                    stg[row * STG_LD + 64] = __ldg(Ly.b_ih + jb) + __ldg(Ly.b_hh + jb);
                }
                tc_fence_before();
                mbar_arrive(ae0 + 8 * acc);
                epi_sync();
                if (et == 0) probe(a, pv, 4);
                constexpr int UPT = 16 / NWQ;  // units per thread
                const int b = et & 63, u0 = (et >> 6) * UPT, j0 = tile * 32 + u0;
                if (b < B) {
                    const long r1 = ((long)t * B + b) * H, r4 = ((long)t * B + b) * 4 * H;
                    // c[t-1] of all this thread's units first: no load waits behind its stores
                    float4 cpv[UPT / 4];
#pragma unroll
                    for (int q4 = 0; q4 < UPT / 4; ++q4)
                        cpv[q4] = t > 0 ? *reinterpret_cast<const float4 *>(Ly.c + r1 - (long)B * H + j0 + 4 * q4)
                                        : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
                    for (int u4 = 0; u4 < UPT; u4 += 4) {
                        const int j = j0 + u4;
                        float gv[4][4];
#pragma unroll
                        for (int g = 0; g < 4; ++g)
#pragma unroll
                            for (int e = 0; e < 4; ++e) {
                                const int gr = g * 32 + u0 + u4 + e;
                                gv[g][e] = stg[gr * STG_LD + b] + stg[gr * STG_LD + 64];
                            }
                        const float cp[4] = {cpv[u4 / 4].x, cpv[u4 / 4].y, cpv[u4 / 4].z, cpv[u4 / 4].w};
                        float ig[4], fg[4], gg[4], og[4], cc[4], hh[4];
#pragma unroll
                        for (int e = 0; e < 4; ++e) {
                            ig[e] = sigm(gv[0][e]);
                            fg[e] = sigm(gv[1][e]);
                            gg[e] = tanhf(gv[2][e]);
                            og[e] = sigm(gv[3][e]);
                            cc[e] = fg[e] * cp[e] + ig[e] * gg[e];
                            hh[e] = og[e] * tanhf(cc[e]);
                        }
                        uint2 p;
                        p.x = pack_bf16(hh[0], hh[1]);
                        p.y = pack_bf16(hh[2], hh[3]);
                        *reinterpret_cast<uint2 *>(Ly.h + r1 + j) = p;
                        *reinterpret_cast<float4 *>(Ly.c + r1 + j) = make_float4(cc[0], cc[1], cc[2], cc[3]);
                        *reinterpret_cast<float4 *>(Ly.gates + r4 + j) = make_float4(ig[0], ig[1], ig[2], ig[3]);
                        *reinterpret_cast<float4 *>(Ly.gates + r4 + H + j) = make_float4(fg[0], fg[1], fg[2], fg[3]);
                        *reinterpret_cast<float4 *>(Ly.gates + r4 + 2 * H + j) = make_float4(gg[0], gg[1], gg[2], gg[3]);
                        *reinterpret_cast<float4 *>(Ly.gates + r4 + 3 * H + j) = make_float4(og[0], og[1], og[2], og[3]);
                    }
                }
            } else {
                // thread = hidden unit (TMEM lane m); this CTA finishes batch rows [hb, hb + 32),
                // this warp rows [hb + 16 half, +16), and swaps the matching 16 columns of the
                // peer's half of its K-partial with the peer CTA
                const int mrow = q * 32 + lane, j = tile * 128 + mrow, hb = rank * 32, c16 = half * 16;
                float mine[16], other[16];
                if (mm) {
                    tmem_ld16(d + hb + c16, mine);
                    tmem_ld16(d + (32 - hb) + c16, other);
                } else {
#pragma unroll
                    for (int i = 0; i < 16; ++i) mine[i] = other[i] = 0.f;
                }
                tc_fence_before();
                mbar_arrive(ae0 + 8 * acc);
                if (ik.n0 + ik.n1 > 0) {
                    const int peer = rank ^ 1;
                    mbar_wait(rempty, eph ^ 1);  // the peer consumed the previous exchange
                    eph ^= 1;
                    const uint32_t dst = mapa_cluster(smem_u32(stg) + (mrow * 32 + c16) * 4, peer);
                    const uint32_t pbar = mapa_cluster(rfull, peer);
#pragma unroll
                    for (int i = 0; i < 4; ++i)
                        asm volatile(
                            "st.async.shared::cluster.mbarrier::complete_tx::bytes.v4.f32 [%0], {%1, %2, %3, %4}, [%5];" ::"r"(
                                dst + i * 16),
                            "f"(other[i * 4]), "f"(other[i * 4 + 1]), "f"(other[i * 4 + 2]), "f"(other[i * 4 + 3]),
                            "r"(pbar)
                            : "memory");
                    if (et == 0) mbar_expect_tx(rfull, 128 * 32 * 4);
                    mbar_wait(rfull, rph);
                    rph ^= 1;
#pragma unroll
                    for (int i = 0; i < 16; ++i) mine[i] += stg[mrow * 32 + c16 + i];
                    epi_sync();  // every thread read its row: hand the buffer back to the peer
                    if (et == 0) probe(a, pv, 4);
                    if (et == 0)
                        asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(
                                         mapa_cluster(rempty, peer))
                                     : "memory");
                }
                const bool top = l == a.L - 1;
                // cell backward over this warp's 16 batch rows, 8 rows at a time: every load of a
                // chunk is issued before any store (the stores may alias the loads as far as the
                // compiler knows, which otherwise serialises one memory latency per row); gates /
                // c were written by the forward launch, so they take the read-only path
                const int hb2 = hb + c16, nb = min(16, B - hb2);
#pragma unroll
                for (int i0 = 0; i0 < 16; i0 += 8) {  // unrolled: mine[] stays in registers
                    if (i0 >= nb) break;
                    float ig[8], fg[8], gg[8], og[8], ct[8], cp[8], dcn[8], dyv[8];
#pragma unroll
                    for (int u = 0; u < 8; ++u) {
                        const int b = hb2 + i0 + u;
                        ig[u] = fg[u] = gg[u] = og[u] = ct[u] = cp[u] = dcn[u] = dyv[u] = 0.f;
                        if (i0 + u < nb) {
                            const long r1 = ((long)t * B + b) * H + j, r4 = ((long)t * B + b) * 4 * H + j;
                            ig[u] = __ldg(Ly.gates + r4);
                            fg[u] = __ldg(Ly.gates + r4 + H);
                            gg[u] = __ldg(Ly.gates + r4 + 2 * H);
                            og[u] = __ldg(Ly.gates + r4 + 3 * H);
                            ct[u] = __ldg(Ly.c + r1);
                            if (t > 0) cp[u] = __ldg(Ly.c + r1 - (long)B * H);
                            if (t < a.T - 1) dcn[u] = Ly.dc[(long)b * H + j];
                            if (top) dyv[u] = __bfloat162float(a.dy_top[r1]);
                        }
                    }
#pragma unroll
                    for (int u = 0; u < 8; ++u) {
                        if (i0 + u >= nb) break;
                        const int b = hb2 + i0 + u;
                        const long r4 = ((long)t * B + b) * 4 * H + j;
                        const float dh = mine[i0 + u] + dyv[u];
                        const float tc = tanhf(ct[u]);
                        const float dct = dh * og[u] * (1.f - tc * tc) + dcn[u];
                        Ly.dc[(long)b * H + j] = dct * fg[u];
                        Ly.da[r4] = __float2bfloat16_rn(dct * gg[u] * ig[u] * (1.f - ig[u]));
                        Ly.da[r4 + H] = __float2bfloat16_rn(dct * cp[u] * fg[u] * (1.f - fg[u]));
                        Ly.da[r4 + 2 * H] = __float2bfloat16_rn(dct * ig[u] * (1.f - gg[u] * gg[u]));
                        Ly.da[r4 + 3 * H] = __float2bfloat16_rn(dh * tc * og[u] * (1.f - og[u]));
                    }
                }
            }
            if (et == 0) probe(a, pv, 6);  // this thread's cell loop done
            epi_sync();
            if (et == 0) {
                probe(a, pv, 7);  // all 128 epilogue threads done
                asm volatile("fence.acq_rel.gpu;" ::: "memory");
                asm volatile("red.relaxed.gpu.global.add.u32 [%0], 1;" ::"l"(a.cnt + l) : "memory");
                probe(a, pv, 5);
            }
            ++pv;
            acc ^= 1;
        }
    }
    tc_fence_before();
    __syncthreads();
    if (BWD) cluster_sync_all();  // no peer st.async / arrive may target an exited CTA
    if (warp == 3) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;" ::"r"(tmem));
}

int wave_smem(bool bwd) { return (bwd ? 8 * STAGE + RECV_BYTES : 7 * STAGE + STG_BYTES) + 256 + 1024; }


int num_sm() {
    static int sms = 0;
    if (!sms) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        if (sms <= 0) sms = 148;
    }
    return sms;
}

// forward: one CTA per item up to one per SM; backward: a CTA pair per item up to one pair
// per two SMs (and no more pairs than can be resident at once)
int wave_grid(int L, int H, bool bwd, int max_pairs) {
    const int items = L * (bwd ? H / 128 : H / 32);
    if (!bwd) return items < num_sm() ? items : num_sm();
    const int pairs = items < max_pairs ? items : max_pairs;
    return 2 * pairs;
}

cudaLaunchConfig_t wave_cfg(bool bwd, int grid, cudaStream_t s, cudaLaunchAttribute *attr) {
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(bwd ? wave_threads<true>() : wave_threads<false>());
    cfg.dynamicSmemBytes = wave_smem(bwd);
    cfg.stream = s;
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = bwd ? 2 : 1;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cfg;
}

int max_pairs_resident() {
    static int n = -1;
    if (n < 0) {
        cudaLaunchAttribute attr[1];
        cudaLaunchConfig_t cfg = wave_cfg(true, 2 * 64, nullptr, attr);
        int c = 0;
        if (cudaOccupancyMaxActiveClusters(&c, lstm_wave_kernel<true>, &cfg) != cudaSuccess) {
            cudaGetLastError();
            c = 0;
        }
        n = c;
    }
    return n;
}

}  // namespace

bool lstm_wave_supported(int L, int B, int H, int I) {
    if (L < 1 || L > LSTM_WAVE_MAX_L || B < 1 || B > 64 || H < 128 || H % 128 || I != H) return false;
    static int ok = 0;
    if (!ok) {
        int n = 0;
        ok = 1;
        if (cudaFuncSetAttribute(lstm_wave_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 wave_smem(false)) != cudaSuccess ||
            cudaFuncSetAttribute(lstm_wave_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 wave_smem(true)) != cudaSuccess ||
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, lstm_wave_kernel<false>, wave_threads<false>(), wave_smem(false)) !=
                cudaSuccess ||
            n < 1 || max_pairs_resident() < 1) {
            cudaGetLastError();
            ok = -1;
        }
    }
    return ok > 0;
}

cudaError_t lstm_wave(const LstmWaveDesc &w, cudaStream_t s) {
    const int L = w.L, H = w.H, T = w.T, B = w.B;
    if (!lstm_wave_supported(L, B, H, H)) return cudaErrorNotSupported;
    WaveArgs a{};
    a.L = L, a.T = T, a.B = B, a.H = H, a.N = (B + 15) / 16 * 16;
    a.tiles = w.bwd ? H / 128 : H / 32;
    a.dy_top = w.dy_top;
    a.cnt = w.cnt;
    WaveMaps m;
    std::memset(&m, 0, sizeof(m));
    const long TB = (long)T * B;
    for (int l = 0; l < L; ++l) {
        a.layer[l] = {w.b_ih[l], w.b_hh[l], w.gates[l], w.c[l], w.h[l], w.da[l], w.dc[l]};
        const int rows = w.bwd ? 64 : 32, cols = 64;
        if (!tma_map_bf16(&m.w_ih[l], w.W_ih[l], H, 4L * H, H, cols, rows) ||
            !tma_map_bf16(&m.w_hh[l], w.W_hh[l], H, 4L * H, H, cols, rows))
            return cudaErrorInvalidValue;
        if (!w.bwd) {
            if (!tma_map_bf16(&m.act[l + 1], w.h[l], H, TB, H, 64, a.N)) return cudaErrorInvalidValue;
        } else if (!tma_map_bf16(&m.act[l], w.da[l], 4L * H, TB, 4L * H, 64, a.N)) {
            return cudaErrorInvalidValue;
        }
    }
    if (!w.bwd && !tma_map_bf16(&m.act[0], w.x, H, TB, H, 64, a.N)) return cudaErrorInvalidValue;
    cudaError_t e = cudaMemsetAsync(w.cnt, 0, sizeof(unsigned) * L, s);
    if (e != cudaSuccess) return e;
    const int grid = wave_grid(L, H, w.bwd, max_pairs_resident());
    {
        // PD_WAVE_L2_MB: MB of the run's weights kept L2-resident (whole layers, evict_last; the
        // rest streams evict_first).  Measured GNMT-8 at N = 1: 0 -> 11.51k, 32 -> 11.80k,
        // 48 -> 11.92k, 64 -> 12.02k, 80 -> 11.97k samples/s; 0 turns the hints off
        const char *e2 = getenv("PD_WAVE_L2_MB");
        const long keep = e2 ? atol(e2) : 64;
        const long per_layer = 2L * 4 * H * H * 2;  // W_ih + W_hh bf16
        a.keep_layers = keep > 0 ? (int)std::min<long>(L, keep * 1000000L / per_layer) : 0;
    }
    // tools only: PD_WAVE_PROBE=<file> appends one line per launch with every CTA's per-visit
    // phase stamps (not while the stream is being captured into a graph)
    static unsigned long long *pbuf = nullptr;
    const char *pfile = getenv("PD_WAVE_PROBE");
    cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
    if (pfile) cudaStreamIsCapturing(s, &cap);
    const size_t pbytes = (size_t)grid * PROBE_V * 8 * sizeof(unsigned long long);
    if (pfile && cap == cudaStreamCaptureStatusNone) {
        if (!pbuf && cudaMalloc(&pbuf, (size_t)1024 * PROBE_V * 8 * sizeof(unsigned long long)) != cudaSuccess)
            pbuf = nullptr;
        if (pbuf && cudaMemsetAsync(pbuf, 0, pbytes, s) == cudaSuccess) a.probe = pbuf;
    }
    cudaLaunchAttribute attr[1];
    cudaLaunchConfig_t cfg = wave_cfg(w.bwd, grid, s, attr);
    ++tl_launches;
    e = w.bwd ? cudaLaunchKernelEx(&cfg, lstm_wave_kernel<true>, m, a)
              : cudaLaunchKernelEx(&cfg, lstm_wave_kernel<false>, m, a);
    if (e == cudaSuccess && a.probe) {
        std::vector<unsigned long long> h(pbytes / 8);
        if (cudaStreamSynchronize(s) == cudaSuccess && cudaMemcpy(h.data(), pbuf, pbytes, cudaMemcpyDeviceToHost) == cudaSuccess) {
            unsigned long long t0 = ~0ull;
            for (auto x : h)
                if (x && x < t0) t0 = x;
            if (FILE *f = fopen(pfile, "a")) {
                fprintf(f, "%s L=%d T=%d B=%d H=%d grid=%d", w.bwd ? "bwd" : "fwd", L, T, B, H, grid);
                for (int c = 0; c < grid; ++c) {
                    fprintf(f, " |");
                    for (int v = 0; v < PROBE_V; ++v) {
                        const unsigned long long *q = &h[((size_t)c * PROBE_V + v) * 8];
                        if (!q[3]) break;
                        for (int ev = 0; ev < 8; ++ev) fprintf(f, " %lld", q[ev] ? (long long)(q[ev] - t0) : -1LL);
                        fprintf(f, " ;");
                    }
                }
                fprintf(f, "\n");
                fclose(f);
            }
        }
    }
    return e;
}

}  // namespace pd
