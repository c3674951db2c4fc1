// pd_internal.h -- internal declarations of libpipedream (not part of the C ABI).
#pragma once

#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <string>
#include <vector>

#include "../../include/pipedream.h"

namespace pd {

// ---------------------------------------------------------------- planner (plan.cpp)
pd_status plan_partition(const pd_layer_profile *layers, int N, int G, const pd_plan_opts *opts, pd_plan_t *out);

// ---------------------------------------------------------------- schedule (schedule.cpp)
// One entry of a worker's static 1F1B-RR op list (R3).
struct Op {
    char kind;  // 'F', 'B', 'U'
    int t;      // global minibatch id
    int j;      // local index of t at this worker (t = replica + j * R_s)
};
// k_s per stage (R2 / R19).  Returns PD_EINVAL for an override on a replicated plan.
pd_status inflight_counts(const pd_plan_t &plan, int depth, std::vector<int> &k);
// F(t_0..t_{k-1}) then (B(t_j) U F(t_{j+k}))* then (B U)* (L1023-1065, L237-241).
std::vector<Op> worker_ops(int R_s, int replica, int k_s, int M);
std::vector<Op> gpipe_ops(bool last_stage, int D, int M);
// receive-ring depth of stage s >= 1: ceil(k_{s-1} R_{s-1} / R_s).
int recv_ring_depth(const pd_plan_t &plan, const std::vector<int> &k, int s);

// ---------------------------------------------------------------- CUDA driver shim (cudadrv.cpp)
struct Driver {
    CUresult (*streamWaitValue32)(CUstream, CUdeviceptr, cuuint32_t, unsigned int) = nullptr;
    CUresult (*tensorMapEncodeTiled)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                     const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                     CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill) = nullptr;
};
const Driver *driver();  // resolved once through cudaGetDriverEntryPoint; nullptr if unavailable

// ---------------------------------------------------------------- kernels
// Per-host-thread launch counter (kernels launched by this library).
extern thread_local uint64_t tl_launches;

enum Major { KMAJ = 0, MNMAJ = 1 };
enum Epi {
    EPI_STORE = 0,  // out = act(acc + bias[n])             (dtype of the path)
    EPI_MASK = 1,   // out = acc * (mask[m][n] > 0)          (dX fused with the ReLU derivative)
    EPI_F32 = 2,    // out(fp32) = acc                       (gradient buffer)
    EPI_SGD = 3,    // master -= lr*acc; slot = cast(master) (fused weight update, bf16 path)
    EPI_ADAM = 4    // Adam on master/m/v; slot = cast(master)
};

// Implicit-GEMM 3x3 convolution on a zero-padded NHWC grid (Hp = H+2, Wp = W+2): GEMM rows
// are padded-grid pixels, K-block kb covers tap kb / kpt and 64 channels (kb % kpt).
struct ConvGeom {
    int taps = 0;          // 9 for fwd / dX, 0 otherwise
    int kpt = 0;           // 64-wide K-blocks per tap
    int a_shift[9] = {};   // A row offset of each tap (fwd: +delta, dX: -delta)
    int b_koff = 0;        // B K-coordinate offset per tap (fwd, K-major weights)
    int b_noff = 0;        // B N-coordinate offset per tap (dX, MN-major weights)
    int b_kshift = 0;      // constant B K-coordinate shift (per-tap dW launch)
    int Hp = 0, Wp = 0;    // padded grid of the OUTPUT rows (epilogue zeroes borders); 0 = off
    int b_tapchunk = 0;    // dW over all 9 taps in one GEMM: B column n = tap*Cp + ci, each 64-column
                           // chunk reads X shifted by a_shift[tap] (value = Cp, multiple of 64; 0 = off)
    int a_inner = 0;       // inner extents of the A / B tensors for the TMA maps (taps > 0)
    int b_inner = 0;
    // packed-tap mode for Cp = 8 inputs (the RGB first layer): the 9 taps' 8-channel slices
    // are packed side by side along K in unswizzled core-matrix layout (one 16-byte TMA box
    // per tap) instead of one mostly-zero 64-wide K-block per tap.
    //   1 = forward (A = X, 9 boxes {8, 128 rows}; B = W [Co][72], 10 boxes {8, Co}; K = 80)
    //   2 = weight gradient (A = dY MN-major; B = X shifted per tap, 9 boxes {8, 64 pixels};
    //       N = 72 (MMA N = 80))
    int c8 = 0;
};

// C(m, n) = sum_k A(m, k) * B(n, k)
//   A(m, k) = amaj == KMAJ ? A[m*lda + k] : A[k*lda + m]
//   B(n, k) = bmaj == KMAJ ? B[n*ldb + k] : B[k*ldb + n]
struct Gemm {
    int M = 0, N = 0, K = 0;
    const void *A = nullptr;
    long lda = 0;
    int amaj = KMAJ;
    const void *B = nullptr;
    long ldb = 0;
    int bmaj = KMAJ;
    int epi = EPI_STORE;
    void *out = nullptr;  // EPI_STORE/MASK: path dtype; EPI_F32: float
    long ldo = 0;
    const float *bias = nullptr;
    int relu = 0;
    const void *mask = nullptr;  // path dtype, ld = ldm
    long ldm = 0;
    // fused update (EPI_SGD / EPI_ADAM), arrays indexed [m*ldo + n]
    float *master = nullptr;
    void *slot = nullptr;  // bf16 new version
    float *adam_m = nullptr, *adam_v = nullptr;
    float lr = 0.f, b1 = 0.f, b2 = 0.f, eps = 0.f;
    int step = 0;
    // optional fp32 scratch for split-K partials (bf16 EPI_STORE / EPI_MASK); nullptr = off
    float *workspace = nullptr;
    long workspace_bytes = 0;
    // the caller keeps `workspace` all-zero between GEMMs: split-K partials are then summed by
    // TMA reduce-add into ONE fp32 tile set (and the reduction kernel re-zeroes what it read)
    int ws_zeroed = 0;
    ConvGeom conv;        // implicit-GEMM convolution (bf16 path only)
    int ksplit = 1;       // explicit split-K (EPI_F32 with atomic_out)
    int max_ctas = 0;     // cap on resident CTAs (0 = every SM): leaves SMs to a concurrent kernel
    int atomic_out = 0;   // EPI_F32: fp32 atomic accumulation into out
    // programmatic dependent launch (cluster split-K path): the kernel may start while the
    // previous kernel of the stream is still running; it loads only B (the weights) before
    // griddepcontrol.wait.  Only for a GEMM whose predecessor is the previous layer's GEMM of
    // the same chain (whose first kernel launched normally), so B is never being written.
    int pdl = 0;
    // wait for a producer kernel running concurrently (EPI_F32 with explicit ksplit): before
    // loading the K-blocks [kb0, kb1) of a unit, wait until *wait_cnt >= (wait_T - kb0*64 /
    // wait_B) * wait_per (acquire) -- rows r of A belong to step r / wait_B, and the producer
    // completes steps in descending order; the splits then run last-rows first
    const unsigned *wait_cnt = nullptr;
    int wait_T = 0, wait_B = 1;
    unsigned wait_per = 0;
};

// cached 2-D bf16 tensor map (128B swizzle), row-major [outer][ld_elems], box {box_inner, box_outer}
bool tma_map_bf16(CUtensorMap *map, const void *base, long inner, long outer, long ld_elems, int box_inner,
                  int box_outer);

// fp32 SIMT GEMM (parity path; no tensor cores, no TF32).  EPI_STORE/MASK/F32 only.
cudaError_t gemm_f32(const Gemm &g, cudaStream_t s);
// bf16 tcgen05/TMEM/TMA GEMM, fp32 accumulation.  All epilogues.
cudaError_t gemm_bf16(const Gemm &g, cudaStream_t s);

// elementwise / reductions (kernels.cu).  T = float or __nv_bfloat16 via `bf16` flag.
cudaError_t col_sum(const void *G, int bf16, long rows, long cols, float *out, cudaStream_t s);
// bias gradient db = column sums of G [rows][cols]; written to grad_out if non-null; if
// master is non-null the SGD/Adam update of the bias is fused (slot receives bf16(master)).
cudaError_t bias_grad(const void *G, int bf16, long rows, long cols, float *grad_out, float *master,
                      __nv_bfloat16 *slot, int opt, float *m, float *v, float lr, float b1, float b2, float eps,
                      int step, cudaStream_t s);
cudaError_t softmax_ce(const void *logits, int bf16, const int32_t *labels, long rows, int C, void *dlogits,
                       float *loss_out, cudaStream_t s);
// out = in - lr * g  (fp32 versions), n elements
cudaError_t sgd_f32(const float *in, const float *g, float *out, long n, float lr, cudaStream_t s);
cudaError_t adam_f32(const float *in, const float *g, float *out, float *m, float *v, long n, float lr, float b1,
                     float b2, float eps, int step, cudaStream_t s);
// bf16 path: master -= lr * g (or Adam), slot = bf16(master).  g may be a replica set:
// g = (sum_r grads[r]) * (1/R), summed in r order (R7).
// grads is a DEVICE array of R pointers; element i of replica r is grads[r][goff + i].
cudaError_t update_master(float *master, __nv_bfloat16 *slot_bf16, float *slot_f32, const float *const *grads,
                          int R, long goff, long n, int opt, float *m, float *v, float lr, float b1, float b2,
                          float eps, int step, cudaStream_t s);
// replica sync of one round, sharded: this replica's parameters [lo, hi) (multiples of 4):
// g = (sum_r grads[r][i]) * (1/R) in r order (R7), optimizer step on w_in[i] (+ m, v), the
// new value stored to out_f32[q][i] and (if out_bf16) bf16 to out_bf16[q][i] for every
// replica q.  grads / out_f32 / out_bf16 are DEVICE arrays of R pointers (peer memory).
cudaError_t update_shard(const float *const *grads, int R, long lo, long hi, const float *w_in, float *const *out_f32,
                         __nv_bfloat16 *const *out_bf16, int nout, int opt, float *m, float *v, float lr, float b1, float b2,
                         float eps, int step, cudaStream_t s);
// bf16 path, one unreplicated fp32 gradient: master -= SGD/Adam step of g, slot = bf16(master);
// vectorised (n % 4 == 0, 16-byte aligned arrays; else cudaErrorInvalidValue)
cudaError_t update_from_grad(float *master, __nv_bfloat16 *slot, const float *g, long n, int opt, float *m, float *v,
                             float lr, float b1, float b2, float eps, int step, cudaStream_t s);
// dst[off[r] + i] = float(src[off[r] + i]) for i < cnt[r], r < n (off, cnt device arrays)
cudaError_t regions_bf16_to_f32(const __nv_bfloat16 *src, float *dst, const long *off, const int *cnt, int n,
                                cudaStream_t s);
cudaError_t f32_to_bf16(const float *in, __nv_bfloat16 *out, long n, cudaStream_t s);
cudaError_t bf16_to_f32(const __nv_bfloat16 *in, float *out, long n, cudaStream_t s);
cudaError_t signal_flag(uint32_t *flag, uint32_t value, cudaStream_t s);
// n elements (bf16 or fp32) uniform in [-scale, scale) from a counter hash of (index, seed)
cudaError_t fill_uniform(void *p, long n, int bf16, float scale, uint32_t seed, cudaStream_t s);

// LSTM / embedding (lstm.cu); `bf16` selects the path dtype of h / dy / da / y / E
cudaError_t lstm_cell_fwd(int bf16, const float *gx, const float *gh, const float *b_ih, const float *b_hh,
                          const float *c_prev, float *gates, float *c_out, void *h_out, void *y_out, int B, int H,
                          cudaStream_t s);
// Persistent weight-stationary LSTM recurrences (lstm_rec.cu, bf16 path): all T steps of one
// layer in ONE launch; W_hh slices stay in shared memory, the step-to-step dependency is a
// per-K-block counter in `cnt` (>= 4H/64 uints, zeroed by the caller before each launch).
//   fwd: gates/c/h[t] from gx[t] (= X W_ih^T, [T][B][4H] fp32) + h[t-1] W_hh^T + b_ih + b_hh
//   bwd: da[t] from dy[t] + da[t+1] W_hh and the saved gates / c (dc carried on chip)
// lstm_rec_supported: shape (H % 256 == 0, H <= 1024, 1 <= B <= 64) and co-residency of the
// clustered grid on this device; callers fall back to the per-step path otherwise.
bool lstm_rec_supported(int B, int H);
cudaError_t lstm_rec_fwd(const float *gx, const float *b_ih, const float *b_hh, const __nv_bfloat16 *Whh,
                         float *gates, float *c, __nv_bfloat16 *h, unsigned *cnt, int T, int B, int H, cudaStream_t s,
                         unsigned long long *probe = nullptr);
cudaError_t lstm_rec_bwd(const __nv_bfloat16 *dy, const float *gates, const float *c, const __nv_bfloat16 *Whh,
                         __nv_bfloat16 *da, unsigned *cnt, int T, int B, int H, cudaStream_t s,
                         unsigned long long *probe = nullptr);
// A stage's stack of L LSTM layers (H = in = out, bf16) as ONE wavefront kernel per direction
// (lstm_wave.cu): the input projection is folded into the per-step GEMM and every layer
// advances one step per wave.  Per layer: weights of the version used, saved state
// (gates / c / h as the per-layer path lays them out), da output, dc scratch [B][H].
constexpr int LSTM_WAVE_MAX_L = 16;
struct LstmWaveDesc {
    int bwd = 0, L = 0, T = 0, B = 0, H = 0;
    const __nv_bfloat16 *x = nullptr;       // forward: input of the bottom layer [T][B][H]
    const __nv_bfloat16 *dy_top = nullptr;  // backward: gradient of the top layer's output
    const __nv_bfloat16 *W_ih[LSTM_WAVE_MAX_L] = {}, *W_hh[LSTM_WAVE_MAX_L] = {};
    const float *b_ih[LSTM_WAVE_MAX_L] = {}, *b_hh[LSTM_WAVE_MAX_L] = {};
    float *gates[LSTM_WAVE_MAX_L] = {}, *c[LSTM_WAVE_MAX_L] = {}, *dc[LSTM_WAVE_MAX_L] = {};
    __nv_bfloat16 *h[LSTM_WAVE_MAX_L] = {}, *da[LSTM_WAVE_MAX_L] = {};
    __nv_bfloat16 *h_out = nullptr;  // forward: second destination of the top layer's h (the stage
                                     // output: the consumer's receive slot, possibly peer memory)
    unsigned *cnt = nullptr;  // >= L uints (zeroed by lstm_wave on the stream)
    // optional residency signal (backward): every CTA of the wave adds 1 to *started (device,
    // zeroed by lstm_wave) when it starts and the last one writes `epoch` to *started_host (device
    // pointer of a mapped pinned host word), so the host can launch work that must not take the
    // wave's SMs before all of them are resident
    unsigned *started = nullptr;
    volatile unsigned *started_host = nullptr;
    unsigned epoch = 0;
};
bool lstm_wave_supported(int L, int B, int H, int I);
// CTAs of the wave launch lstm_wave would issue for an L-layer run (H hidden units); *cl =
// its cluster K-split (a layer's timestep counts as done at cnt >= (done steps) * (H/128) * cl)
int lstm_wave_grid(bool bwd, int L, int H, int *cl = nullptr);
cudaError_t lstm_wave(const LstmWaveDesc &w, cudaStream_t s);
cudaError_t lstm_cell_bwd(int bf16, const void *dy, const float *dh_rec, const float *gates, const float *c,
                          const float *c_prev, float *dc, void *da, int B, int H, cudaStream_t s);
cudaError_t embedding_fwd(int bf16, const int32_t *tok, const void *E, void *y, long rows, int H, cudaStream_t s);
cudaError_t embedding_bwd(int bf16, const int32_t *tok, const void *dy, float *dE, long rows, int H, cudaStream_t s);

// conv / pool on the zero-padded NHWC layout (conv.cu)
cudaError_t pad_nhwc(const float *in, void *out, int bf16, int B, int H, int W, int C, int Cp, cudaStream_t s);
cudaError_t pool_fwd(int bf16, const void *x, void *y, int B, int H, int W, int C, int out_padded, cudaStream_t s);
cudaError_t pool_bwd(int bf16, const void *x, const void *dy, void *dx, int B, int H, int W, int C, int dy_padded,
                     int mask_relu, cudaStream_t s);
cudaError_t col_sum_tall(const void *G, int bf16, long rows, int cols, float *out, cudaStream_t s);
cudaError_t conv_fwd_f32(const float *x, const float *Wd, const float *bias, float *y, int B, int H, int W, int Cp,
                         int Cout, int relu, cudaStream_t s);
cudaError_t conv_dx_f32(const float *dy, const float *Wd, const float *xmask, float *dx, int B, int H, int W, int Cp,
                        int Cout, cudaStream_t s);
cudaError_t conv_dw_f32(const float *dy, const float *x, float *dW, int B, int H, int W, int Cp, int Cout,
                        cudaStream_t s);

}  // namespace pd
