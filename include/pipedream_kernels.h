/*
 * pipedream_kernels.h -- kernel-level entry points of libpipedream.so, for kernel parity
 * tests and micro-benchmarks.  Same conventions as pipedream.h, except that every pointer
 * here is a DEVICE pointer owned by the caller and the call is asynchronous on `stream`
 * (a cudaStream_t passed as void*; NULL = legacy default stream).
 */
#ifndef PIPEDREAM_KERNELS_H
#define PIPEDREAM_KERNELS_H

#include "pipedream.h"

#ifdef __cplusplus
extern "C" {
#endif

/* C(m, n) = sum_k A(m, k) B(n, k) for 0 <= m < M, 0 <= n < N, 0 <= k < K, fp32 accumulation.
 *   A(m, k) = a_mn_major ? A[k*lda + m] : A[m*lda + k]      (row-major storage, element units)
 *   B(n, k) = b_mn_major ? B[k*ldb + n] : B[n*ldb + k]
 * This one contraction is the forward (X W^T), input gradient (G W) and weight gradient
 * (G^T X) of a linear layer; the epilogue is fused:
 *   PD_EPI_STORE  out[m*ldo+n] = act(C + bias[n])            (dtype of the path)
 *   PD_EPI_MASK   out[m*ldo+n] = C * (mask[m*ldm+n] > 0)     (ReLU derivative from its output)
 *   PD_EPI_F32    out[m*ldo+n] = C                           (fp32, e.g. replica gradients)
 *   PD_EPI_SGD    master[i] -= lr*C; slot[i] = bf16(master[i]), i = m*ldo+n  (bf16 only)
 *   PD_EPI_ADAM   Adam(step) on master/adam_m/adam_v; slot[i] = bf16(master[i]) (bf16 only)
 * dtype PD_BF16 runs the tcgen05/TMEM/TMA kernel (A, B, out, mask, slot bf16; rows 16-byte
 * aligned); PD_FP32 the SIMT fp32 kernel (STORE/MASK/F32 only).
 * Errors: PD_EINVAL (bad sizes/epilogue), PD_ECUDA (launch failure). */
typedef enum { PD_EPI_STORE = 0, PD_EPI_MASK = 1, PD_EPI_F32 = 2, PD_EPI_SGD = 3, PD_EPI_ADAM = 4 } pd_epilogue;

typedef struct {
    int dtype;
    int M, N, K;
    const void *A;
    long lda;
    int a_mn_major;
    const void *B;
    long ldb;
    int b_mn_major;
    int epilogue;
    void *out;
    long ldo;
    const float *bias;
    int relu;
    const void *mask;
    long ldm;
    float *master;
    void *slot;
    float *adam_m, *adam_v;
    float lr, beta1, beta2, eps;
    int step;
    float *workspace;      /* optional fp32 scratch (device) for split-K partial sums of small-M
                              STORE/MASK GEMMs (bf16); NULL disables split-K           */
    long workspace_bytes;
    int workspace_zeroed;  /* 1: the caller guarantees `workspace` is all-zero on entry; split-K
                              partials are then summed by TMA reduce-add (fp32, in L2) into ONE
                              M x N set, and the workspace is all-zero again when the GEMM's
                              last kernel completes (the summation order of the splits is not
                              fixed).  0: partials stored per split, summed in split order */
} pd_gemm_desc;

PD_API pd_status pd_kernel_gemm(const pd_gemm_desc *g, void *stream);

/* Mean softmax cross-entropy over `rows` rows of C logits (dtype of the path), labels int32;
 * dlogits = (softmax - onehot) / rows; *loss (device fp32) += mean loss. */
PD_API pd_status pd_kernel_softmax_ce(int dtype, const void *logits, const int32_t *labels, long rows, int C,
                                      void *dlogits, float *loss, void *stream);

/* Bias gradient db[c] = sum_r G[r][c] over `rows` rows of a row-major [rows][cols] output
 * gradient G (dtype of the path) -- the db = sum dY of the backward pass (PAPER.md L1145-1161,
 * SURVEY §8(a) a7) -- either written to grad_out (device fp32 [cols]) or, when `master` is
 * given (bf16 path), applied as the optimizer step of a10 to the latest weights: master -= SGD
 * or Adam step (m, v fp32, bias-corrected with `step`), slot_bf16 = bf16(master).  Sums are in
 * a fixed order (deterministic).  Device pointers; PD_EINVAL on bad sizes/pointers. */
PD_API pd_status pd_kernel_bias_grad(int dtype, const void *G, long rows, long cols, float *grad_out, float *master,
                                     void *slot_bf16, int optimizer, float *m, float *v, float lr, float beta1,
                                     float beta2, float eps, int step, void *stream);

/* The recurrent half of one LSTM layer (bf16 path, R22: PyTorch form, gates i, f, g,
 * o; h0 = c0 = 0), all T steps in ONE persistent launch (csrc/lstm_rec.cu): W_hh stays in
 * shared memory, step t waits only for the K-blocks of h[t-1] (da[t+1]) it multiplies.
 *   direction 0 (forward):  a = gx[t] + b_ih + b_hh + h[t-1] W_hh^T  (gx = X W_ih^T, fp32
 *       [T][B][4H]) -> gates fp32 [T][B][4H] (sigmoid/tanh activations i, f, g, o),
 *       c fp32 [T][B][H], h bf16 [T][B][H]        (LSTM-gate layers)
 *   direction 1 (backward through time): dh = dy[t] + da[t+1] W_hh; cell backward with the
 *       saved gates / c -> da bf16 [T][B][4H] (pre-activation gate gradients; dc carried on
 *       chip)                                       (row a7)
 * w_hh: bf16 [4H][H] (the weight version the op uses).  counters: device uint32 scratch of at
 * least 4H/64 entries, zeroed by this call on `stream`.  probe: optional device uint64
 * [grid][T][8] %globaltimer phase stamps (tools/lstm_probe.py), NULL = off.
 * All pointers are DEVICE pointers owned by the caller; asynchronous on `stream`.
 * Errors: PD_EUNSUPPORTED (H % 256 != 0, H > 1024, B > 64, or the clustered grid cannot be
 * co-resident on this GPU), PD_EINVAL (null pointer / bad direction), PD_ECUDA. */
typedef struct {
    int direction;
    int T, B, H;
    const float *gx, *b_ih, *b_hh;
    const void *w_hh;
    float *gates, *c;
    void *h;
    const void *dy;
    void *da;
    unsigned *counters;
    unsigned long long *probe;
} pd_lstm_rec_desc;

PD_API pd_status pd_kernel_lstm_rec(const pd_lstm_rec_desc *d, void *stream);

#ifdef __cplusplus
}
#endif
#endif
