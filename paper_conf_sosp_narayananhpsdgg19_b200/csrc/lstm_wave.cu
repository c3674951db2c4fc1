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

constexpr int ATILE = 128 * 128;         // [128 rows][64 K] bf16 (or 2 x [64 K][64 rows] MN-major)
constexpr int BTILE = 64 * 128;          // [<= 64 rows][64 K] bf16
constexpr int STAGE = ATILE + BTILE;

// Cluster K-split (CL CTAs per item, template parameter): the CTAs of a cluster split an
// item's K-blocks, and each finishes R = 64 / CL of the 64 accumulator columns (batch rows,
// on the 64-column grid: columns >= B are padding nobody uses).  Partials travel to the
// owning CTA through DSMEM (st.async + mbarrier complete_tx) into its exchange buffer
// xbuf[source slot][128 rows][row stride]:
//   forward (CL 1 or 2): one slot per CTA of the cluster (own partial staged locally), row
//                        stride R + 1 floats (bank-conflict-free staging stores by TMEM
//                        row and cell-loop reads by hidden unit); the
//                        forward's b_ih + b_hh per gate row in a separate 128-float array
//   backward (CL 2, 4, 8): CL - 1 slots (own partial stays in registers), stride R
// More CTAs per item = fewer weight / activation bytes each CTA ingests per wave (the per-SM
// ingest, not the tensor pipe, bounds a wave), so short runs (a pipeline stage's 2-3 layers)
// spread each wave over the whole machine.
template <bool BWD, int CL>
struct WaveCfg {
    static constexpr int S = BWD ? 8 : 7;  // operand ring stages
    static constexpr int R = 64 / CL;      // accumulator columns (batch rows) a CTA finishes
    static constexpr int RP = BWD ? R : R + 1;  // forward: odd stride, conflict-free by row and by unit
    static constexpr int SLOTS = BWD ? CL - 1 : CL;
    static constexpr int XBYTES = (SLOTS > 0 ? SLOTS : 1) * 128 * RP * 4;
    static constexpr int BIAS_BYTES = BWD ? 0 : 128 * 4;
    // forward, CL = 2: the peer's chunk is staged here and moved by one bulk DSMEM copy
    static constexpr int OUT_BYTES = (!BWD && CL > 1) ? 128 * RP * 4 : 0;
    static constexpr int SMEM = S * STAGE + XBYTES + BIAS_BYTES + OUT_BYTES + 256 + 1024;
    static_assert(64 % CL == 0 && (BWD ? (CL >= 2 && R / 2 >= 4) : CL <= 2), "unsupported cluster split");
};

// NC consecutive fp32 columns of this warp's 32 TMEM lanes (NC = 4, 8, 16), waited
template <int NC>
__device__ __forceinline__ void tmem_ldn(uint32_t taddr, float (&v)[NC]) {
    uint32_t r[NC];
    if constexpr (NC == 16) {
        asm volatile(
            "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
            : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
              "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
            : "r"(taddr));
    } else if constexpr (NC == 8) {
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                     : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
                     : "r"(taddr));
    } else {
        static_assert(NC == 4, "tmem_ldn: 4, 8 or 16 columns");
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0,%1,%2,%3}, [%4];"
                     : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3])
                     : "r"(taddr));
    }
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
    for (int i = 0; i < NC; ++i) v[i] = __uint_as_float(r[i]);
}

__device__ __forceinline__ void st_async_v4(uint32_t dst, const float *v, uint32_t bar) {
    asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.v4.f32 [%0], {%1, %2, %3, %4}, [%5];" ::"r"(dst),
                 "f"(v[0]), "f"(v[1]), "f"(v[2]), "f"(v[3]), "r"(bar)
                 : "memory");
}
__device__ __forceinline__ void arrive_remote(uint32_t bar_local, int rank) {
    asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(mapa_cluster(bar_local, rank))
                 : "memory");
}

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
    __nv_bfloat16 *h2;         // forward: optional second destination of h (top layer: the stage output)
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
    unsigned *started;            // optional residency signal (LstmWaveDesc::started)
    volatile unsigned *started_host;
    unsigned epoch;
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
constexpr int WAVE_THREADS = 384;

// SIG: the residency signal (WaveArgs::started) is compiled in only where a caller asks for it --
// the few instructions at the top measured 4.5 % slower waves when present in every instantiation
template <bool BWD, int CL, bool SIG = false>
__global__ void __launch_bounds__(WAVE_THREADS, 1) lstm_wave_kernel(const __grid_constant__ WaveMaps m, const WaveArgs a) {
    constexpr int NE = WAVE_THREADS - 128;  // epilogue threads
    using WC = WaveCfg<BWD, CL>;
    constexpr int S = WC::S, R = WC::R, RP = WC::RP;
    auto epi_sync = [] { epi_sync_n<NE>(); };
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *sm = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    float *xbuf = reinterpret_cast<float *>(sm + S * STAGE);                 // exchange / staging
    float *sbias = reinterpret_cast<float *>(sm + S * STAGE + WC::XBYTES);  // forward biases
    float *outbox = reinterpret_cast<float *>(sm + S * STAGE + WC::XBYTES + WC::BIAS_BYTES);  // fwd, CL = 2
    uint64_t *bars = reinterpret_cast<uint64_t *>(sm + S * STAGE + WC::XBYTES + WC::BIAS_BYTES + WC::OUT_BYTES);
    // bars: full_w[S], full_x[S], empty[S], acc_full[2], acc_empty[2], recv_full, recv_empty
    const uint32_t fw0 = smem_u32(bars), fx0 = smem_u32(bars + S), em0 = smem_u32(bars + 2 * S);
    const uint32_t af0 = smem_u32(bars + 3 * S), ae0 = smem_u32(bars + 3 * S + 2);
    const uint32_t rfull = smem_u32(bars + 3 * S + 4), rempty = smem_u32(bars + 3 * S + 5);
    uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(bars + 3 * S + 6);
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int H = a.H, B = a.B, N = a.N;
    const int rank = CL > 1 ? (int)cluster_rank() : 0;

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
        mbar_init(rempty, CL > 1 ? CL - 1 : 1);  // every peer that receives from this CTA releases
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 3) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 128;" ::"r"(smem_u32(tmem_slot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    tc_fence_before();
    __syncthreads();
    if (CL > 1) cluster_sync_all();  // the peers' barriers exist before any remote arrive / st.async
    tc_fence_after();
    const uint32_t tmem = *tmem_slot;
    if (SIG && tid == 0) {  // this CTA is resident; the last one tells the host
        if (atomicAdd(a.started, 1u) == gridDim.x - 1) {
            __threadfence_system();
            *a.started_host = a.epoch;
            __threadfence_system();
        }
    }
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
        const int half = (warp - 4) >> 2;  // which half of this CTA's columns (backward) / chunks (forward)
        const int et = tid - 128;
        const uint32_t xb = smem_u32(xbuf);
        ItemIter<CL> it;
        int l, tile, t, acc = 0, pv = 0;
        uint32_t aph[2] = {0, 0}, rph = 0, eph = 0;
        while (it.next(a, BWD, l, tile, t)) {
            const ItemK ik = item_k(a, BWD, l, t, rank, CL);
            const bool mm = ik.hi > ik.lo;
            // while the MMA runs, load this thread's cell inputs (they do not depend on the
            // accumulator): forward c[t-1] of its units; backward (one row chunk per thread,
            // CL >= 4) the saved gates, c[t], c[t-1], the dc carry and the top layer's dy --
            // for CL = 2 (two chunks, no registers to spare) only pulled into L2
            constexpr bool PRE_B = BWD && R / 2 <= 8;
            constexpr int PR = PRE_B ? R / 2 : 1, FC = BWD ? 1 : R / 8;
            float pig[PR], pfg[PR], pgg[PR], pog[PR], pct[PR], pcp[PR], pdc[PR], pdy[PR];
            float fcp[FC];
            if constexpr (BWD) {
                const WaveLayer &Lp = a.layer[l];
                if constexpr (PRE_B) {
                    const int j = tile * 128 + q * 32 + lane, hb2 = rank * R + half * (R / 2);
                    const bool top = l == a.L - 1;
#pragma unroll
                    for (int u = 0; u < PR; ++u) {
                        const int b = hb2 + u;
                        pig[u] = pfg[u] = pgg[u] = pog[u] = pct[u] = pcp[u] = pdc[u] = pdy[u] = 0.f;
                        if (b < B) {
                            const long r1 = ((long)t * B + b) * H + j, r4 = ((long)t * B + b) * 4 * H + j;
                            pig[u] = __ldg(Lp.gates + r4);
                            pfg[u] = __ldg(Lp.gates + r4 + H);
                            pgg[u] = __ldg(Lp.gates + r4 + 2 * H);
                            pog[u] = __ldg(Lp.gates + r4 + 3 * H);
                            pct[u] = __ldg(Lp.c + r1);
                            if (t > 0) pcp[u] = __ldg(Lp.c + r1 - (long)B * H);
                            if (t < a.T - 1) pdc[u] = Lp.dc[(long)b * H + j];
                            if (top) pdy[u] = __bfloat162float(a.dy_top[r1]);
                        }
                    }
                } else {
                    // lane i of warp q fetches the 128-byte lines of batch row rank * R + i
                    const int b = rank * R + lane, jq = tile * 128 + q * 32;
                    if (half == 0 && lane < R && b < B) {
                        const long r1 = ((long)t * B + b) * H + jq, r4 = ((long)t * B + b) * 4 * H + jq;
#pragma unroll
                        for (int g = 0; g < 4; ++g)
                            asm volatile("prefetch.global.L2 [%0];" ::"l"(Lp.gates + r4 + (long)g * H));
                        asm volatile("prefetch.global.L2 [%0];" ::"l"(Lp.c + r1));
                        if (t > 0) asm volatile("prefetch.global.L2 [%0];" ::"l"(Lp.c + r1 - (long)B * H));
                        if (t < a.T - 1) asm volatile("prefetch.global.L2 [%0];" ::"l"(Lp.dc + (long)b * H + jq));
                    }
                }
            } else {
                // forward cell mapping: lane = hidden unit, warp w covers rows w, w + 8, ...
                const int j = tile * 32 + lane;
#pragma unroll
                for (int i = 0; i < FC; ++i) {
                    const int b = rank * R + (et >> 5) + 8 * i;
                    fcp[i] = (t > 0 && b < B) ? a.layer[l].c[((long)(t - 1) * B + b) * H + j] : 0.f;
                }
            }
            mbar_wait(af0 + 8 * acc, aph[acc]);
            aph[acc] ^= 1;
            tc_fence_after();
            if (et == 0) probe(a, pv, 3);
            const uint32_t d = tmem + acc * 64 + ((uint32_t)(q * 32) << 16);
            const WaveLayer &Ly = a.layer[l];
            if constexpr (!BWD) {
                // stage D[row = g*32 + u][b] so one thread sees all four gates of (u, b): chunk ch
                // (accumulator columns 32 ch .. 32 ch + 31) belongs to CTA ch of a pair (CL = 2)
                // or to this CTA (CL = 1); it lands in the owner's slot `rank`
                const int row = q * 32 + lane;
                constexpr int NWQ = NE / 128;  // epilogue warps per TMEM lane quadrant
                if (CL > 1) {
                    mbar_wait(rempty, eph ^ 1);  // the peer has consumed what we sent it last item
                    eph ^= 1;
                }
#pragma unroll
                for (int ch = half; ch < 2; ch += NWQ) {
                    float v[32];
                    tmem_ld32(d + ch * 32, v);
                    const int owner = CL == 1 ? 0 : ch;
                    // own chunk: straight into this CTA's slot; the peer's: into the outbox
                    const uint32_t base = owner == rank ? xb + (uint32_t)((rank * 128 + row) * RP * 4) +
                                                              (CL == 1 ? ch * 32 * 4 : 0)
                                                        : smem_u32(outbox) + (uint32_t)(row * RP * 4);
#pragma unroll
                    for (int i = 0; i < 32; ++i)
                        asm volatile("st.shared.f32 [%0], %1;" ::"r"(base + i * 4), "f"(v[i]) : "memory");
                }
                if (CL > 1) fence_proxy_async();  // the outbox, written by this thread, feeds a bulk copy
                // gate row `row` = g*32 + u: b_ih + b_hh, so the cell loop reads biases from smem
                if (half == 0) {
                    const int gi = row >> 5, uu = row & 31, jb = gi * H + tile * 32 + uu;
                    sbias[row] = __ldg(Ly.b_ih + jb) + __ldg(Ly.b_hh + jb);
                }
                tc_fence_before();
                mbar_arrive(ae0 + 8 * acc);
                if (CL > 1) {
                    // the whole outbox to the peer's slot `rank` in one bulk DSMEM copy
                    epi_sync();
                    if (et == 0) {
                        const int peer = rank ^ 1;
                        constexpr uint32_t bytes = 128 * RP * 4;
                        asm volatile(
                            "cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                                mapa_cluster(xb + (uint32_t)(rank * 128 * RP * 4), peer)),
                            "r"(smem_u32(outbox)), "r"(bytes), "r"(mapa_cluster(rfull, peer))
                            : "memory");
                        mbar_expect_tx(rfull, bytes);
                    }
                    mbar_wait(rfull, rph);
                    rph ^= 1;
                }
                epi_sync();
                if (et == 0) probe(a, pv, 4);
                // cell: lane = hidden unit u (coalesced loads / stores along H), warp w = et / 32
                // covers this CTA's rows w, w + 8, ... (R / 8 of them)
                const int u = lane, j = tile * 32 + u;
#pragma unroll
                for (int i = 0; i < R / 8; ++i) {
                    const int br = (et >> 5) + 8 * i, b = rank * R + br;
                    if (b >= B) break;
                    float gv[4];
#pragma unroll
                    for (int g = 0; g < 4; ++g) {
                        const int gr = g * 32 + u;
                        float x = sbias[gr];
#pragma unroll
                        for (int src = 0; src < CL; ++src) x += xbuf[(src * 128 + gr) * RP + br];
                        gv[g] = x;
                    }
                    const float ig = sigm(gv[0]), fg = sigm(gv[1]), gg = tanhf(gv[2]), og = sigm(gv[3]);
                    const float cc = fg * fcp[i] + ig * gg, hh = og * tanhf(cc);
                    const long r1 = ((long)t * B + b) * H + j, r4 = ((long)t * B + b) * 4 * H + j;
                    const __nv_bfloat16 hb16 = __float2bfloat16_rn(hh);
                    Ly.h[r1] = hb16;
                    if (Ly.h2) Ly.h2[r1] = hb16;
                    Ly.c[r1] = cc;
                    Ly.gates[r4] = ig;
                    Ly.gates[r4 + H] = fg;
                    Ly.gates[r4 + 2 * H] = gg;
                    Ly.gates[r4 + 3 * H] = og;
                }
            } else {
                // thread = hidden unit (TMEM lane m); this CTA finishes batch rows [hb, hb + R),
                // this warp the RH rows [hb + c0, hb + c0 + RH); the matching RH columns of every
                // peer's share go to that peer (its slot for this CTA), and this CTA's own
                // columns collect the CL - 1 partials the peers send
                constexpr int RH = R / 2, RC = RH < 8 ? RH : 8;
                const int mrow = q * 32 + lane, j = tile * 128 + mrow, hb = rank * R, c0 = half * RH;
                float mine[RH];
                if (mm) {
                    tmem_ldn<RH>(d + hb + c0, mine);
                } else {
#pragma unroll
                    for (int i = 0; i < RH; ++i) mine[i] = 0.f;
                }
                const bool exch = ik.n0 + ik.n1 > 0;  // the same for every CTA of the cluster
                if (exch) {
                    mbar_wait(rempty, eph ^ 1);  // every peer consumed what we sent it last item
                    eph ^= 1;
#pragma unroll
                    for (int pr = 0; pr < CL; ++pr) {
                        if (pr == rank) continue;
                        float other[RH];
                        if (mm) {
                            tmem_ldn<RH>(d + pr * R + c0, other);
                        } else {
#pragma unroll
                            for (int i = 0; i < RH; ++i) other[i] = 0.f;
                        }
                        const int slot = rank < pr ? rank : rank - 1;
                        const uint32_t dst = mapa_cluster(xb + (uint32_t)(((slot * 128 + mrow) * R + c0) * 4), pr);
                        const uint32_t pbar = mapa_cluster(rfull, pr);
#pragma unroll
                        for (int i = 0; i < RH / 4; ++i) st_async_v4(dst + i * 16, other + i * 4, pbar);
                    }
                }
                tc_fence_before();
                mbar_arrive(ae0 + 8 * acc);
                if (exch) {
                    if (et == 0) mbar_expect_tx(rfull, (uint32_t)(CL - 1) * 128 * R * 4);
                    mbar_wait(rfull, rph);
                    rph ^= 1;
#pragma unroll
                    for (int sl = 0; sl < CL - 1; ++sl)
#pragma unroll
                        for (int i = 0; i < RH; ++i) mine[i] += xbuf[(sl * 128 + mrow) * R + c0 + i];
                    epi_sync();  // every thread read its row: hand the buffers back to the peers
                    if (et == 0) probe(a, pv, 4);
                    if (et == 0)
                        for (int pr = 0; pr < CL; ++pr)
                            if (pr != rank) arrive_remote(rempty, pr);
                }
                // cell backward over this warp's RH batch rows
                const int hb2 = hb + c0, nb = min(RH, B - hb2);
                auto cell = [&](int u, float dh, float ig, float fg, float gg, float og, float ct, float cp, float dcn) {
                    const int b = hb2 + u;
                    const long r4 = ((long)t * B + b) * 4 * H + j;
                    const float tc = tanhf(ct);
                    const float dct = dh * og * (1.f - tc * tc) + dcn;
                    Ly.dc[(long)b * H + j] = dct * fg;
                    Ly.da[r4] = __float2bfloat16_rn(dct * gg * ig * (1.f - ig));
                    Ly.da[r4 + H] = __float2bfloat16_rn(dct * cp * fg * (1.f - fg));
                    Ly.da[r4 + 2 * H] = __float2bfloat16_rn(dct * ig * (1.f - gg * gg));
                    Ly.da[r4 + 3 * H] = __float2bfloat16_rn(dh * tc * og * (1.f - og));
                };
                if constexpr (PRE_B) {
#pragma unroll
                    for (int u = 0; u < RH; ++u)
                        if (u < nb) cell(u, mine[u] + pdy[u], pig[u], pfg[u], pgg[u], pog[u], pct[u], pcp[u], pdc[u]);
                } else {
                    const bool top = l == a.L - 1;
                    // RC rows at a time: every load of a chunk is issued before any store (the
                    // stores may alias the loads as far as the compiler knows, which otherwise
                    // serialises one memory latency per row); gates / c were written by the
                    // forward launch, so they take the read-only path
#pragma unroll
                    for (int i0 = 0; i0 < RH; i0 += RC) {  // unrolled: mine[] stays in registers
                        if (i0 >= nb) break;
                        float ig[RC], fg[RC], gg[RC], og[RC], ct[RC], cp[RC], dcn[RC], dyv[RC];
#pragma unroll
                        for (int u = 0; u < RC; ++u) {
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
                        for (int u = 0; u < RC; ++u) {
                            if (i0 + u >= nb) break;
                            cell(i0 + u, mine[i0 + u] + dyv[u], ig[u], fg[u], gg[u], og[u], ct[u], cp[u], dcn[u]);
                        }
                    }
                }
            }
            if (et == 0) probe(a, pv, 6);  // this thread's cell loop done
            epi_sync();
            if (et == 0) {
                // forward, CL = 2: the cell loop above read the peer's slot -- release it
                if (!BWD && CL > 1)
                    for (int pr = 0; pr < CL; ++pr)
                        if (pr != rank) arrive_remote(rempty, pr);
                probe(a, pv, 7);  // all epilogue threads done
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
    if (CL > 1) cluster_sync_all();  // no peer st.async / arrive may target an exited CTA
    if (warp == 3) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;" ::"r"(tmem));
}

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

template <bool BWD, int CL>
cudaLaunchConfig_t wave_cfg(int grid, cudaStream_t s, cudaLaunchAttribute *attr) {
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(WAVE_THREADS);
    cfg.dynamicSmemBytes = WaveCfg<BWD, CL>::SMEM;
    cfg.stream = s;
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = CL;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cfg;
}

// clusters of this instantiation that can be resident at once (0 if it cannot launch); the
// wavefront's spin-waits need every CTA of the grid resident, so grids never exceed this
template <bool BWD, int CL>
int max_clusters() {
    static int n = -1;
    if (n < 0) {
        n = 0;
        if (cudaFuncSetAttribute(lstm_wave_kernel<BWD, CL>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 WaveCfg<BWD, CL>::SMEM) == cudaSuccess) {
            cudaLaunchAttribute attr[1];
            cudaLaunchConfig_t cfg = wave_cfg<BWD, CL>(CL * 64, nullptr, attr);
            int c = 0;
            if (cudaOccupancyMaxActiveClusters(&c, lstm_wave_kernel<BWD, CL>, &cfg) == cudaSuccess) n = c;
        }
        cudaGetLastError();
    }
    return n;
}

int max_clusters(bool bwd, int cl) {
    if (!bwd) return cl == 2 ? max_clusters<false, 2>() : max_clusters<false, 1>();
    return cl == 8 ? max_clusters<true, 8>() : cl == 4 ? max_clusters<true, 4>() : max_clusters<true, 2>();
}

// Cluster size: the widest K-split whose clusters all fit at once with one item each (every
// SM ingesting a 1/CL share of an item per wave); when the items outnumber the resident
// clusters (long runs), the narrowest split (forward 1, backward 2: the whole machine is busy
// anyway and fewer, larger shares exchange less).
int choose_cl(bool bwd, int items) {
    const int sms = num_sm();
    const int cands[2][3] = {{2, 1, 1}, {8, 4, 2}};
    for (int cl : cands[bwd]) {
        const int mc = max_clusters(bwd, cl);
        if (mc >= items && cl * items <= sms) return cl;
    }
    return bwd ? 2 : 1;
}

}  // namespace

int lstm_wave_grid(bool bwd, int L, int H, int *cl_out) {
    const int items = L * (bwd ? H / 128 : H / 32);
    const int cl = choose_cl(bwd, items);
    if (cl_out) *cl_out = cl;
    return cl * std::min(items, max_clusters(bwd, cl));
}

bool lstm_wave_supported(int L, int B, int H, int I) {
    if (L < 1 || L > LSTM_WAVE_MAX_L || B < 1 || B > 64 || H < 128 || H % 128 || I != H) return false;
    return max_clusters(false, 1) >= 1 && max_clusters(true, 2) >= 1;
}

// the smallest wave grid that runs every item: CL CTAs per item up to the resident clusters
template <bool BWD, int CL, bool SIG = false>
cudaError_t launch_wave(const WaveMaps &m, const WaveArgs &a, int items, cudaStream_t s) {
    const int mc = max_clusters<BWD, CL>();
    if (mc < 1) return cudaErrorNotSupported;
    const int clusters = items < mc ? items : mc;
    cudaLaunchAttribute attr[1];
    cudaLaunchConfig_t cfg = wave_cfg<BWD, CL>(CL * clusters, s, attr);
    ++tl_launches;
    if (SIG) {
        static bool attr = false;  // (max_clusters set the attribute of the SIG = false twin)
        if (!attr) {
            const cudaError_t e = cudaFuncSetAttribute(lstm_wave_kernel<BWD, CL, true>,
                                                       cudaFuncAttributeMaxDynamicSharedMemorySize, WaveCfg<BWD, CL>::SMEM);
            if (e != cudaSuccess) return e;
            attr = true;
        }
    }
    return cudaLaunchKernelEx(&cfg, lstm_wave_kernel<BWD, CL, SIG>, m, a);
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
        a.layer[l] = {w.b_ih[l], w.b_hh[l], w.gates[l], w.c[l], w.h[l], l == L - 1 ? w.h_out : nullptr, w.da[l], w.dc[l]};
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
    a.started = w.started;
    a.started_host = w.started_host;
    a.epoch = w.epoch;
    if (w.started && (e = cudaMemsetAsync(w.started, 0, sizeof(unsigned), s)) != cudaSuccess) return e;
    const int items = L * a.tiles;
    const int cl = choose_cl(w.bwd, items);
    const int grid = cl * std::min(items, max_clusters(w.bwd, cl));
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
    if (!w.bwd) e = cl == 2 ? launch_wave<false, 2>(m, a, items, s) : launch_wave<false, 1>(m, a, items, s);
    else if (a.started && a.started_host) e = cl == 8 ? launch_wave<true, 8, true>(m, a, items, s)
                          : cl == 4 ? launch_wave<true, 4, true>(m, a, items, s)
                                    : launch_wave<true, 2, true>(m, a, items, s);
    else if (cl == 8) e = launch_wave<true, 8>(m, a, items, s);
    else if (cl == 4) e = launch_wave<true, 4>(m, a, items, s);
    else e = launch_wave<true, 2>(m, a, items, s);
    if (e == cudaSuccess && a.probe) {
        std::vector<unsigned long long> h(pbytes / 8);
        if (cudaStreamSynchronize(s) == cudaSuccess && cudaMemcpy(h.data(), pbuf, pbytes, cudaMemcpyDeviceToHost) == cudaSuccess) {
            unsigned long long t0 = ~0ull;
            for (auto x : h)
                if (x && x < t0) t0 = x;
            if (FILE *f = fopen(pfile, "a")) {
                fprintf(f, "%s L=%d T=%d B=%d H=%d grid=%d CL=%d max_clusters fwd1/2 %d/%d bwd2/4/8 %d/%d/%d",
                        w.bwd ? "bwd" : "fwd", L, T, B, H, grid, cl, max_clusters(false, 1), max_clusters(false, 2),
                        max_clusters(true, 2), max_clusters(true, 4), max_clusters(true, 8));
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
