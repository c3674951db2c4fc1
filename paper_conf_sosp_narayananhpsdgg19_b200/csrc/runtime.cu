// runtime.cu -- the 1F1B-RR pipeline runtime with weight stashing (§3.2-3.3, §4).
//
// One host thread per local worker (stage s, replica r) walks the worker's static op list
// (schedule.cpp) and issues its kernels on the worker's own CUDA stream, so issue order is
// execution order (the event trace is exact).  Cross-worker dependencies are the only
// synchronisation (the schedule is static, "without expensive distributed coordination",
// L1083-1085):
//   activation  F(s-1, t) -> F(s, t)   the producing GEMM writes straight into the consumer's
//                                      receive-ring slot (peer pointer over NVLink when the
//                                      consumer is another GPU), then posts the link;
//   gradient    B(s+1, t) -> B(s, t)   the first layer's dX GEMM writes into the upstream
//                                      worker's gradient ring slot, then posts;
//   replicas    round j of a replicated stage: every replica posts "gradient ready", each
//               replica reduces all R gradients (replica order, R7) in one fused
//               reduce+update kernel reading peer memory, then posts "read done".
// A link is an event ring + host counters when both ends live in this process (every wait
// refers to an already-issued record, so any hardware-queue mapping is deadlock free), or
// a flag word in the consumer's memory written by a release-store kernel and awaited with
// cuStreamWaitValue32 when the ends are in different processes (CUDA IPC).
//
// State per worker (§4 "Parameter State" / "Intermediate State", L1337-1371):
//   weight-stash ring   k_s versions; version v lives in slot v mod k_s.  F reads the
//                       latest, B reads the stashed v(s,t); the update writes version v+1
//                       into slot (v+1) mod k_s -- the slot of the oldest version, which no
//                       pending backward references any more.
//                       No copies: stashing a version is remembering its index.
//   fp32 master + Adam  bf16 path only the master is fp32 (R21); optimizer state is not
//                       versioned (R9).
//   receive rings       activations D_s deep (they double as the first layer's stash),
//                       gradients k_s deep; slot = local index mod depth.
//   activation stash    inputs of the stage's inner layers, k_s deep.
#include <algorithm>
#include <atomic>
#include <chrono>
#include <cmath>
#include <condition_variable>
#include <cstdio>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

#include "pd_internal.h"

using namespace pd;

namespace {

// ---------------------------------------------------------------- errors
struct CudaFail {
    cudaError_t e;
    const char *what;
};
#define CK(x)                                              \
    do {                                                   \
        cudaError_t _e = (x);                              \
        if (_e != cudaSuccess) throw CudaFail{_e, #x};     \
    } while (0)
struct Abort {};
struct SlotViolation {
    std::string msg;
};

long numel_params(const pd_layer_desc &d) {
    switch (d.kind) {
    case PD_LINEAR: return (long)d.out * d.in + d.out;
    case PD_LSTM: return 4L * d.out * d.in + 4L * d.out * d.out + 8L * d.out;
    case PD_CONV3X3: return (long)d.out * d.in * 9 + d.out;
    case PD_MAXPOOL2: return 0;
    case PD_EMBEDDING: return (long)d.in * d.out;
    }
    return -1;
}
long rows_of(const pd_layer_desc &d, int B) { return d.seq_len > 0 ? (long)d.seq_len * B : (long)B; }
long in_elems(const pd_layer_desc &d, int B) {
    switch (d.kind) {
    case PD_LINEAR: return rows_of(d, B) * d.in;
    case PD_LSTM: return (long)d.seq_len * B * d.in;
    case PD_CONV3X3:
    case PD_MAXPOOL2: return (long)B * d.height * d.width * d.in;
    case PD_EMBEDDING: return (long)d.seq_len * B;
    }
    return 0;
}
long out_elems(const pd_layer_desc &d, int B) {
    switch (d.kind) {
    case PD_LINEAR: return rows_of(d, B) * d.out;
    case PD_LSTM: return (long)d.seq_len * B * d.out;
    case PD_CONV3X3: return (long)B * d.height * d.width * d.out;
    case PD_MAXPOOL2: return (long)B * (d.height / 2) * (d.width / 2) * d.in;
    case PD_EMBEDDING: return (long)d.seq_len * B * d.out;
    }
    return 0;
}

// Device layouts.  Conv / pool inputs live on a zero-padded NHWC grid [B][H+2][W+2][Cp]
// (Cp = channels rounded up to 8 for conv inputs, so rows are 16-byte aligned for TMA);
// everything else is the contract layout.  A layer writes its output in the layout of the
// layer that consumes it.
int cpad8(int c) { return (c + 7) / 8 * 8; }
bool padded_in(const pd_layer_desc &d) { return d.kind == PD_CONV3X3 || d.kind == PD_MAXPOOL2; }
int dev_channels(const pd_layer_desc &d) { return d.kind == PD_CONV3X3 ? cpad8(d.in) : d.in; }
long dev_in_elems(const std::vector<pd_layer_desc> &L, int l, int B) {
    const pd_layer_desc &d = L[l];
    if (padded_in(d)) return (long)B * (d.height + 2) * (d.width + 2) * dev_channels(d);
    return in_elems(d, B);
}
long dev_out_elems(const std::vector<pd_layer_desc> &L, int l, int B) {
    return l + 1 < (int)L.size() ? dev_in_elems(L, l + 1, B) : out_elems(L[l], B);
}
// device parameter count (conv weights are stored [Cout][3][3][Cp], K-major for the GEMM)
long dev_params(const pd_layer_desc &d) {
    if (d.kind == PD_CONV3X3) return (long)d.out * 9 * cpad8(d.in) + d.out;
    return numel_params(d);
}
// contract layout <-> device layout of one layer's parameters (host side)
void params_to_dev(const pd_layer_desc &d, const float *src, float *dst) {
    if (d.kind != PD_CONV3X3) {
        std::memcpy(dst, src, sizeof(float) * numel_params(d));
        return;
    }
    const int Ci = d.in, Cp = cpad8(d.in), Co = d.out;
    for (int co = 0; co < Co; ++co)
        for (int tap = 0; tap < 9; ++tap)
            for (int ci = 0; ci < Cp; ++ci)
                dst[((long)co * 9 + tap) * Cp + ci] = ci < Ci ? src[((long)co * Ci + ci) * 9 + tap] : 0.f;
    std::memcpy(dst + (long)Co * 9 * Cp, src + (long)Co * Ci * 9, sizeof(float) * Co);
}
void params_from_dev(const pd_layer_desc &d, const float *src, float *dst) {
    if (d.kind != PD_CONV3X3) {
        std::memcpy(dst, src, sizeof(float) * numel_params(d));
        return;
    }
    const int Ci = d.in, Cp = cpad8(d.in), Co = d.out;
    for (int co = 0; co < Co; ++co)
        for (int ci = 0; ci < Ci; ++ci)
            for (int tap = 0; tap < 9; ++tap) dst[((long)co * Ci + ci) * 9 + tap] = src[((long)co * 9 + tap) * Cp + ci];
    std::memcpy(dst + (long)Co * Ci * 9, src + (long)Co * 9 * Cp, sizeof(float) * Co);
}

// ---------------------------------------------------------------- links
enum LinkType { L_ACT = 0, L_GRAD = 1, L_READY = 2, L_DONE = 3 };

struct Link {
    bool remote = false;
    // local (same process): event ring + host counters
    std::mutex mu;
    std::condition_variable cv;
    int64_t posted = 0, waited = 0;
    std::vector<cudaEvent_t> ev;
    int device = -1;  // producer's device (events are created there)
    // remote (other process): flag in the consumer's memory
    uint32_t *remote_flag = nullptr;  // producer side, IPC-mapped
    uint32_t *local_flag = nullptr;   // consumer side
    int64_t rposted = 0;              // producer: messages posted over all runs
    int64_t rbase = 0, rcount = 0;    // consumer: messages of earlier runs / the producer posts this run
                                      // (static: known from the schedule, not from what was awaited)
    // slot-ownership checker (local links): the producer's vector clock at each post
    std::vector<std::vector<int32_t>> snap;
};

// ---------------------------------------------------------------- IPC blob
constexpr int MAX_SYNC_SLOTS = 32;  // weight-stash slots a replicated worker exposes to its peers
struct IpcBlob {
    uint32_t magic;
    int32_t stage, replica, device;
    int32_t has_recv, has_grad, has_rgrad;
    cudaIpcMemHandle_t recv, grad, rgrad0, rgrad1, flags;
    // replicated stages: the weight-stash slots and the fp32 master, which the peers' sharded
    // updates write (replica sync as reduce-scatter -> update -> all-gather)
    int32_t nslots, has_master;
    cudaIpcMemHandle_t wslot[MAX_SYNC_SLOTS], master;
};
constexpr uint32_t BLOB_MAGIC = 0x50443032u;  // "PD02"

// Buffers a worker exposes to others (local pointers, or IPC-mapped in this process).
struct Shared {
    void *recv = nullptr;      // activation receive ring (stage > 0)
    void *grad = nullptr;      // gradient receive ring (stage < n-1)
    float *rgrad[2] = {};      // replica gradient buffers (R_s > 1), round parity
    void *wslot[MAX_SYNC_SLOTS] = {};  // replicated stages: weight-stash slots (peers write their shards)
    int nslots = 0;
    float *master = nullptr;   // replicated stages, bf16 path: fp32 master (peers write their shards)
    uint32_t *flags = nullptr; // flag words (remote links)
    bool valid = false;
    bool standin = false;      // pd_stage_solo: local buffers standing in for an absent worker
};

struct Worker;

}  // namespace

struct pd_ctx {
    pd_plan_t plan{};
    std::vector<pd_layer_desc> layers;
    pd_train_cfg cfg{};
    int n = 0;                       // stages
    int nw = 0;                      // workers
    std::vector<int> wbase;          // first worker id per stage
    std::vector<int> kdef;           // default k_s
    std::vector<int> kalloc;         // allocated stash depth (max over default and max_depth)
    std::vector<int> Dalloc, Galloc; // ring depths as allocated
    std::vector<long> poff;          // parameter offset of each layer inside its stage buffer
    std::vector<long> pcount;        // parameter count of each layer in the device layout
    std::vector<long> hcount;        // ... in the contract layout (pd_stage_init / pd_get_params)
    std::vector<std::unique_ptr<Worker>> W;  // by worker id (null when remote)
    std::vector<Shared> shared;              // by worker id
    std::map<std::tuple<int, int, int>, std::unique_ptr<Link>> links;  // (type, src, dst)
    int esz = 4;                     // element size of the path dtype
    int n_data = 0;
    // results of the last run
    int last_M = 0;
    std::vector<int32_t> vmap;
    double host_ms = 0;
    // op index of F / B / U of local index j in worker w's static list of this run (checker)
    std::vector<std::vector<int32_t>> opF, opB, opU;
    int ktime_mask = 0xFF;           // kernel classes timed when record_trace >= 2
    int layer_prof = 0;              // per-layer F / B device times (pd_set_layer_profiling)
    std::vector<void *> solo_bufs;   // pd_stage_solo stand-in buffers (owned)
    std::mutex done_mu;              // worker threads of a pd_run finishing (watchdog wake-up)
    std::condition_variable done_cv;
    int running = 0;
    std::atomic<bool> abort{false};
    std::mutex err_mu;
    pd_status sticky = PD_OK;
    std::string err;

    void fail(pd_status s, const std::string &msg) {
        std::lock_guard<std::mutex> g(err_mu);
        if (sticky == PD_OK) {
            sticky = s;
            err = msg;
        }
        abort = true;
        for (auto &kv : links) {
            std::lock_guard<std::mutex> lg(kv.second->mu);
            kv.second->cv.notify_all();
        }
    }
    int worker_id(int s, int r) const { return wbase[s] + r; }
    int stage_of(int w) const {
        int s = 0;
        while (s + 1 < n && wbase[s + 1] <= w) ++s;
        return s;
    }
    int flag_index(int type, int src_stage, int src_rep, int dst_stage) const;
    int flag_count(int s) const;
};

namespace {

struct Worker {
    pd_ctx *ctx;
    int id, stage, replica, device;
    int first, last;   // layer range
    long P = 0;        // parameters of the stage
    int k = 1;         // stash slots allocated
    int D = 0, G = 0;  // receive ring depths
    cudaStream_t stream = nullptr;
    cudaStream_t side = nullptr;           // second stream: dW+update overlapping the next dX
    std::vector<cudaEvent_t> ev_dx, ev_dw; // per stage layer, reused by every backward
    cudaEvent_t ev_fork = nullptr;         // main -> side fork at the start of an overlapped backward
    // weights
    std::vector<void *> wslot;  // k versions (path dtype)
    float *master = nullptr;    // bf16 path
    // vertical sync, bf16 path: fp32 biases of the version a forward uses (from its bf16
    // slot), bias regions (offset, count) of the stage's layers on the device
    float *fbias = nullptr;
    long *breg_off = nullptr;
    int *breg_cnt = nullptr;
    int n_breg = 0;
    float *adam_m = nullptr, *adam_v = nullptr;
    float *gbuf = nullptr;      // fp32 gradient (unreplicated fp32 path / biases)
    float *ws = nullptr;        // split-K partials of the bf16 GEMMs
    long ws_bytes = 0;
    float *rgrad[2] = {};       // replicated stages: gradient per round parity
    const float **rgrad_ptrs = nullptr;  // device array [2][R]: peers' rgrad for each parity
    // sharded replica sync: device arrays of every replica's destinations of a new version --
    // sync_f32[slot][R]: fp32 masters (bf16 path, same for every slot) or fp32 slot `slot`;
    // sync_bf16[slot][R]: bf16 slot `slot` (bf16 path)
    float **sync_f32 = nullptr;
    __nv_bfloat16 **sync_bf16 = nullptr;
    const float **self_grad_ptr = nullptr;  // device array [1]: gbuf
    // GPipe flush schedule (PD_SYNC_GPIPE): one fp32 gradient buffer per minibatch of a flush
    // group (gp_grad[i] for the group's i-th minibatch), their device pointer array, and the
    // update's destinations per weight slot (fp32: master on the bf16 path / slot q; bf16: slot q)
    std::vector<float *> gp_grad;
    const float **gp_ptrs = nullptr;
    float **gp_out_f32 = nullptr;
    __nv_bfloat16 **gp_out_bf16 = nullptr;
    // activations
    std::vector<void *> act;     // per inner layer l (index l-first, l>first): k slots of in_elems
    void *recv = nullptr;        // D slots (stage > 0)
    void *gring = nullptr;       // G slots (stage < n-1)
    void *scratch[3] = {};       // dY rotation (3 deep so a dW on the side stream can still read it)
    void *logits = nullptr, *dlogits = nullptr;  // last stage
    void *data_in = nullptr;     // stage 0: n_data inputs (path dtype)
    int32_t *tokens = nullptr;   // stage 0 embedding
    int32_t *labels = nullptr;   // last stage
    // LSTM layers: per layer a k-deep ring of saved state {gates fp32 [T*B][4H], c fp32
    // [T*B][H], h (path dtype) [T*B][H]}; per worker transient scratch for the recurrence
    std::vector<void *> aux;     // index l - first (nullptr for other kinds)
    std::vector<long> aux_bytes;
    float *lstm_gx = nullptr, *lstm_gh = nullptr, *lstm_dh = nullptr, *lstm_dc = nullptr;
    void *lstm_da = nullptr;
    unsigned *lstm_cnt = nullptr;  // step counters of the persistent recurrence kernels
    void *lstm_wda = nullptr;      // wavefront backward: da of every layer of an LSTM run
    int lstm_wmax = 0;             // ... for runs of up to this many layers
    float *lstm_wdc = nullptr;     // ... and their dc carries
    // weight gradients of a short wavefront run computed while its backward wave runs (one
    // stream + completion event per GEMM: 2 per layer, runs of <= 3 layers)
    cudaStream_t dw_stream[6] = {};
    cudaEvent_t dw_ev[6] = {};
    unsigned *wave_flag = nullptr;  // mapped pinned host word: the backward wave is resident (epoch)
    unsigned wave_epoch = 0;
    int lstm_rec = -1;             // persistent recurrences usable (-1 = not decided yet)
    // CUDA graphs of the LSTM recurrences (T steps of small GEMM + cell kernels), keyed by
    // (layer, direction, saved-state slot, weight slot, dY pointer): replayed instead of
    // re-issuing ~3T launches per layer
    std::map<std::tuple<int, int, int, int, const void *>, std::pair<cudaGraphExec_t, int>> graphs;
    // whole-op graphs (F / B of an all-linear bf16 SGD stage), keyed by every pointer the op uses
    std::map<std::vector<uintptr_t>, std::pair<cudaGraphExec_t, int>> opgraphs;
    float *loss_scratch = nullptr;  // CE writes here inside a graph; copied to losses[t] after
    float *stage_in = nullptr;   // fp32 upload staging for pd_set_data (bf16 path)
    long stage_in_elems = 0;
    float *losses = nullptr;     // last stage, per minibatch of the run
    int losses_cap = 0;
    uint32_t *flags = nullptr;
    // bookkeeping
    int version = 0;
    int run_base = 0;  // version at the start of the current pd_run (equal on every stage)
    std::map<int, int> fwd_version;  // local index -> version used by its forward
    std::vector<pd_event> events;
    std::vector<std::pair<cudaEvent_t, cudaEvent_t>> op_ev;  // record_trace 2
    std::vector<cudaEvent_t> ev_pool;
    cudaEvent_t run_ev[2] = {nullptr, nullptr};  // start / end of this worker's part of a run
    std::vector<std::pair<cudaEvent_t, cudaEvent_t>> kev[PD_KERNEL_CLASSES];  // per kernel class (record_trace 2)
    struct LayerEv {
        int layer;
        char dir;  // 'F' or 'B'
        cudaEvent_t a, b;
    };
    std::vector<LayerEv> lev;  // layer profiling: one per layer per F / B op
    uint64_t launches = 0;
    uint64_t bytes_sent = 0;
    uint64_t replica_bytes = 0;  // peer bytes of the sharded replica sync (gradient reads + pushes)
    int updates_total = 0;  // Adam step counter base (persists across runs)
    // slot-ownership checker: vc[w] = number of ops of worker w known (through the messages
    // this worker has awaited, transitively) to be complete before this worker's current op;
    // vc[id] counts this worker's own ops
    std::vector<int32_t> vc;
    std::vector<char> wave_inner;  // per stage layer: inside an LSTM wavefront run (input = saved h below)
    // watchdog state (pd_run reports a run that makes no progress): the op being issued and
    // where the host thread is -- 0 issuing, 1 waiting for ring space in link_post, 2 waiting
    // for a message in link_wait, 3 synchronising at the end of the run, 4 finished
    std::atomic<int> st_op{-1}, st_where{4};
    std::atomic<long> st_link{0};

    ~Worker();
};

Worker::~Worker() {
    if (device >= 0) cudaSetDevice(device);
    if (stream) cudaStreamSynchronize(stream);
    for (void *p : wslot) cudaFree(p);
    for (void *p : gp_grad) cudaFree(p);
    for (void *p : act) cudaFree(p);
    for (void *p : aux)
        if (p) cudaFree(p);
    void *lb[] = {lstm_gx, lstm_gh, lstm_dh, lstm_dc, lstm_da, lstm_cnt, lstm_wda, lstm_wdc};
    for (void *p : lb)
        if (p) cudaFree(p);
    void *bufs[] = {master, fbias, (void *)breg_off, (void *)breg_cnt, adam_m, adam_v, gbuf, ws, stage_in, rgrad[0], rgrad[1], recv, gring, scratch[0], scratch[1], scratch[2], logits,
                    dlogits, data_in, tokens, labels, losses, flags, (void *)rgrad_ptrs, (void *)self_grad_ptr,
                    (void *)sync_f32, (void *)sync_bf16, (void *)gp_ptrs, (void *)gp_out_f32, (void *)gp_out_bf16};
    for (void *p : bufs)
        if (p) cudaFree(p);
    for (cudaEvent_t e : ev_pool) cudaEventDestroy(e);
    for (cudaEvent_t e : run_ev)
        if (e) cudaEventDestroy(e);
    for (auto &kv : graphs) cudaGraphExecDestroy(kv.second.first);
    for (auto &kv : opgraphs) cudaGraphExecDestroy(kv.second.first);
    if (loss_scratch) cudaFree(loss_scratch);
    for (cudaEvent_t e : ev_dx) cudaEventDestroy(e);
    for (int i = 0; i < 6; ++i) {
        if (dw_ev[i]) cudaEventDestroy(dw_ev[i]);
        if (dw_stream[i]) cudaStreamDestroy(dw_stream[i]);
    }
    if (wave_flag) cudaFreeHost(wave_flag);
    for (cudaEvent_t e : ev_dw) cudaEventDestroy(e);
    if (ev_fork) cudaEventDestroy(ev_fork);
    if (side) cudaStreamDestroy(side);
    if (stream) cudaStreamDestroy(stream);
}

size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

template <typename T>
T *dalloc(size_t bytes) {
    void *p = nullptr;
    if (bytes == 0) bytes = 16;
    cudaError_t e = cudaMalloc(&p, align_up(bytes, 256));
    if (e != cudaSuccess) throw CudaFail{e, "cudaMalloc"};
    // The zero fill runs on the legacy stream, which does NOT order with the workers'
    // non-blocking streams: complete it before anyone else touches the buffer.
    CK(cudaMemset(p, 0, align_up(bytes, 256)));
    CK(cudaDeviceSynchronize());
    return static_cast<T *>(p);
}

}  // namespace

// Flag words of the consumer worker of stage `dst_stage`:
//   [0, R_{s-1})                       activation from producer replica p   (L_ACT)
//   [R_{s-1}, R_{s-1}+R_{s+1})         gradient from downstream replica c   (L_GRAD)
//   then R_s "ready" and R_s "done" words from each peer replica           (L_READY / L_DONE)
int pd_ctx::flag_index(int type, int src_stage, int src_rep, int dst_stage) const {
    const int s = dst_stage;
    const int rp = s > 0 ? plan.stage[s - 1].replicas : 0;
    const int rn = s + 1 < n ? plan.stage[s + 1].replicas : 0;
    const int rs = plan.stage[s].replicas;
    (void)src_stage;
    switch (type) {
    case L_ACT: return src_rep;
    case L_GRAD: return rp + src_rep;
    case L_READY: return rp + rn + src_rep;
    case L_DONE: return rp + rn + rs + src_rep;
    }
    return -1;
}
int pd_ctx::flag_count(int s) const {
    const int rp = s > 0 ? plan.stage[s - 1].replicas : 0;
    const int rn = s + 1 < n ? plan.stage[s + 1].replicas : 0;
    return rp + rn + 2 * plan.stage[s].replicas;
}

namespace {

// ---------------------------------------------------------------- link operations
Link &get_link(pd_ctx *c, int type, int src, int dst) {
    auto key = std::make_tuple(type, src, dst);
    auto it = c->links.find(key);
    if (it == c->links.end()) throw CudaFail{cudaErrorInvalidValue, "missing link"};
    return *it->second;
}

thread_local Worker *tl_worker = nullptr;  // the worker this host thread runs (watchdog state)

// `vc`: the posting worker's vector clock (snapshotted with the message, local links only)
void link_post(pd_ctx *c, Link &L, cudaStream_t s, const std::vector<int32_t> &vc) {
    if (L.remote) {
        ++L.rposted;
        CK(signal_flag(L.remote_flag, (uint32_t)L.rposted, s));
        return;
    }
    const int E = (int)L.ev.size();
    if (tl_worker) tl_worker->st_where = 1, tl_worker->st_link = L.posted;
    {
        std::unique_lock<std::mutex> g(L.mu);
        L.cv.wait(g, [&] { return L.posted - L.waited < E || c->abort.load(); });
        if (c->abort) throw Abort{};
    }
    if (tl_worker) tl_worker->st_where = 0;
    CK(cudaEventRecord(L.ev[L.posted % E], s));
    {
        std::lock_guard<std::mutex> g(L.mu);
        L.snap[L.posted % E] = vc;
        ++L.posted;
    }
    L.cv.notify_all();
}

// Message idx of this run (idx < 0: the previous runs' messages -- every one of them).  The
// waiting worker's vector clock absorbs the producer's snapshot (local links).
void link_wait(pd_ctx *c, Link &L, cudaStream_t s, int64_t idx, std::vector<int32_t> &vc) {
    if (L.remote) {
        // flags are never reset: run r's message idx is value rbase + idx + 1
        const int64_t want = idx < 0 ? L.rbase : L.rbase + idx + 1;
        if (want <= 0) return;
        CUresult r = driver()->streamWaitValue32(s, (CUdeviceptr)L.local_flag, (cuuint32_t)want,
                                                 CU_STREAM_WAIT_VALUE_GEQ);
        if (r != CUDA_SUCCESS) throw CudaFail{cudaErrorUnknown, "cuStreamWaitValue32"};
        return;
    }
    if (idx < 0) return;  // same process: the previous pd_run joined every worker's stream
    const int E = (int)L.ev.size();
    if (tl_worker) tl_worker->st_where = 2, tl_worker->st_link = idx;
    {
        std::unique_lock<std::mutex> g(L.mu);
        L.cv.wait(g, [&] { return L.posted > idx || c->abort.load(); });
        if (c->abort) throw Abort{};
    }
    if (tl_worker) tl_worker->st_where = 0;
    CK(cudaStreamWaitEvent(s, L.ev[idx % E], 0));
    {
        std::lock_guard<std::mutex> g(L.mu);
        const std::vector<int32_t> &sn = L.snap[idx % E];
        for (size_t i = 0; i < sn.size() && i < vc.size(); ++i) vc[i] = std::max(vc[i], sn[i]);
        if (L.waited < idx + 1) L.waited = idx + 1;
    }
    L.cv.notify_all();
}

// ---------------------------------------------------------------- layer kernels
struct LayerCtx {
    pd_ctx *c;
    Worker *w;
    int bf16;
};

const void *elem_ptr(const void *base, long idx, int esz) { return static_cast<const char *>(base) + idx * esz; }
void *elem_ptr(void *base, long idx, int esz) { return static_cast<char *>(base) + idx * esz; }

cudaError_t run_gemm(int bf16, const Gemm &g, cudaStream_t s) { return bf16 ? gemm_bf16(g, s) : gemm_f32(g, s); }

// y = act(x W^T + b)
void linear_forward(const LayerCtx &L, const pd_layer_desc &d, const void *W, const float *bias_f32, const void *x,
                    void *y, float *ws, long ws_bytes, int pdl = 0) {
    const int B = L.c->cfg.minibatch;
    Gemm g;
    g.M = (int)rows_of(d, B);
    g.N = d.out;
    g.K = d.in;
    g.A = x;
    g.lda = d.in;
    g.amaj = KMAJ;
    g.B = W;
    g.ldb = d.in;
    g.bmaj = KMAJ;
    g.epi = EPI_STORE;
    g.out = y;
    g.ldo = d.out;
    g.bias = bias_f32;
    g.relu = d.act == PD_ACT_RELU;
    g.workspace = ws;
    g.workspace_bytes = ws_bytes;
    g.pdl = pdl;
    CK(run_gemm(L.bf16, g, L.w->stream));
}

}  // namespace

// ---------------------------------------------------------------- worker execution
namespace {

struct Exec {
    pd_ctx *c;
    Worker *w;
    int M;
    std::vector<int> k;  // in-flight counts of this run
    int bf16;
    int esz;
    bool timing;
    int ev_used = 0;

    const pd_layer_desc &layer(int l) const { return c->layers[l]; }
    int B() const { return c->cfg.minibatch; }
    bool gpipe() const { return c->cfg.sync_mode == PD_SYNC_GPIPE; }  // flush groups of k[0] (R27)
    int n() const { return c->n; }

    // weights of layer l in stash slot `slot` (path dtype)
    void *Wl(int l, int slot) const { return elem_ptr(w->wslot[slot], c->poff[l], esz); }
    // fp32 bias of layer l: the master (bf16 path) or the slot itself (fp32 path)
    const float *bias_f32(int l, int slot) const {
        const pd_layer_desc &d = layer(l);
        const long off = c->poff[l] + (long)d.out * d.in;
        return fwd_f32(off, slot);
    }
    // fp32 view of forward parameters at offset `off` of version slot `slot`: the slot itself
    // (fp32 path); on the bf16 path the fp32 master (= latest, weight stashing) or the
    // slot's biases widened to fp32 (vertical sync, where F may use an older version)
    const float *fwd_f32(long off, int slot) const {
        if (!bf16) return static_cast<const float *>(w->wslot[slot]) + off;
        return (w->fbias ? w->fbias : w->master) + off;
    }

    // input of layer l for local index j
    const void *layer_input(int l, int t, int j) const {
        const pd_layer_desc &d = layer(l);
        if (l > w->first && w->wave_inner[l - w->first]) return lstm_state(l - 1, j).h;
        if (l == w->first) {
            if (w->stage == 0) {
                const int di = t % c->n_data;
                if (d.kind == PD_EMBEDDING) return w->tokens + (long)di * in_elems(d, B());
                return elem_ptr(w->data_in, (long)di * dev_in_elems(c->layers, l, B()), esz);
            }
            return elem_ptr(w->recv, (long)(j % w->D) * dev_in_elems(c->layers, l, B()), esz);
        }
        return elem_ptr(w->act[l - w->first], (long)(j % w->k) * dev_in_elems(c->layers, l, B()), esz);
    }

    // timing events: the pre-sized pool, grown on demand (never while capturing: the callers
    // return before asking for one then)
    cudaEvent_t pool_event() {
        if (ev_used >= (int)w->ev_pool.size()) {
            cudaEvent_t e;
            CK(cudaEventCreate(&e));
            w->ev_pool.push_back(e);
        }
        return w->ev_pool[ev_used++];
    }
    // per-kernel-class device time (pd_stats.kern_ms classes)
    bool capturing = false;
    cudaEvent_t kstart(int cls) {
        if (capturing || !timing || !((c->ktime_mask >> cls) & 1)) return nullptr;
        cudaEvent_t a = pool_event();
        CK(cudaEventRecord(a, w->stream));
        return a;
    }
    void kend(int cls, cudaEvent_t a) {
        if (!a) return;
        cudaEvent_t b = pool_event();
        CK(cudaEventRecord(b, w->stream));
        w->kev[cls].push_back({a, b});
    }
    // layer profiling (the self-profiler's T_l, L841-843): events around each layer's share of
    // an F or B op; the op then runs serialised on the worker's stream (no side stream, no graphs)
    cudaEvent_t lstart() {
        if (!c->layer_prof || capturing) return nullptr;
        cudaEvent_t a = pool_event();
        CK(cudaEventRecord(a, w->stream));
        return a;
    }
    void lend(int l, char dir, cudaEvent_t a) {
        if (!a) return;
        cudaEvent_t b = pool_event();
        CK(cudaEventRecord(b, w->stream));
        w->lev.push_back({l, dir, a, b});
    }
    void record_start() {
        if (!timing) return;
        cudaEvent_t a = pool_event();
        CK(cudaEventRecord(a, w->stream));
        w->op_ev.push_back({a, nullptr});
    }
    void record_end() {
        if (!timing) return;
        cudaEvent_t b = pool_event();
        CK(cudaEventRecord(b, w->stream));
        w->op_ev.back().second = b;
    }
    void trace(char kind, int mb, int vin, int vout) {
        if (!c->cfg.record_trace) return;
        pd_event e{};
        e.worker = (int16_t)w->id;
        e.stage = (int16_t)w->stage;
        e.replica = (int16_t)w->replica;
        e.kind = kind;
        e.seq = (int32_t)w->events.size();
        e.minibatch = mb;
        e.version_in = vin;
        e.version_out = vout;
        e.start_us = e.end_us = NAN;
        w->events.push_back(e);
    }

    // ---------------- slot ownership (L1349-1353)
    // A ring slot may be rewritten only once the op that last reads its previous content is
    // known to be complete: `other`'s op (F/B/U list `opl`, local index jo) must be in this
    // worker's vector clock, i.e. some message this worker awaited was posted after it (every
    // post is the last action of an op, stream-ordered after all of the op's kernels).  A
    // violation is a schedule / ring-depth bug: the run fails with PD_ESTATE.  Only workers of
    // this process are checked (remote clocks do not travel with the flag words).
    void hb_require(int other, const std::vector<std::vector<int32_t>> &opl, int jo, const char *what, int t) {
        if (jo < 0 || other == w->id || !c->W[other] || jo >= (int)opl[other].size()) return;
        const int op = opl[other][jo];
        if (w->vc[other] > op) return;
        char buf[320];
        snprintf(buf, sizeof buf,
                 "slot ownership: worker %d, minibatch %d: %s (op %d of worker %d is not known to be complete)",
                 w->id, t, what, op, other);
        throw SlotViolation{buf};
    }
    // the weight slot a backward's update writes holds no version a pending backward still uses
    void check_weight_slot(int nslot, int j, int t) {
        for (const auto &kv : w->fwd_version)
            if (kv.first != j && kv.second % w->k == nslot) {
                char buf[256];
                snprintf(buf, sizeof buf,
                         "slot ownership: worker %d, minibatch %d: update would overwrite version %d (slot %d) "
                         "still stashed for local minibatch %d",
                         w->id, t, kv.second, nslot, kv.first);
                throw SlotViolation{buf};
            }
    }

    // ---------------- F(s, t)
    void forward(int t, int j) {
        const int s = w->stage;
        if (s > 0) {
            const int p = t % c->plan.stage[s - 1].replicas;
            const int src = c->worker_id(s - 1, p);
            Link &L = get_link(c, L_ACT, src, w->id);
            // message index on this link: minibatches from p to this replica before t
            link_wait(c, L, w->stream, act_msg_index(s - 1, t), w->vc);
            hb_require(src, c->opF, t / c->plan.stage[s - 1].replicas, "activation used before its forward", t);
        }
        // weight stashing: the latest version.  Vertical sync: the tag the input stage gave t,
        // its latest version at F(0,t) = base + max(0, t - k_0 + 1) on the static schedule
        // (L1180-1186; base = the version every stage had when this pd_run started)
        const bool vsync = c->cfg.sync_mode == PD_SYNC_VERTICAL;
        const int v = vsync ? w->run_base + std::max(0, t - k[0] + 1) : w->version;
        if (v > w->version || v <= w->version - w->k)
            throw CudaFail{cudaErrorInvalidValue, "vertical sync: tagged version not in the stash ring"};
        const int slot = v % w->k;
        w->fwd_version[j] = v;
        if (c->cfg.record_trace) c->vmap[(long)s * M + t] = v;
        trace('F', t, v, v);
        record_start();
        void *y_last = w->logits;
        if (s + 1 < n()) {
            const int Rn = c->plan.stage[s + 1].replicas;
            const int cw = c->worker_id(s + 1, t % Rn);
            const int jc = t / Rn;
            hb_require(cw, c->opB, jc - c->Dalloc[s + 1],
                       "activation receive slot rewritten before the backward that reads it", t);
            y_last = elem_ptr(c->shared[cw].recv, (long)(jc % c->Dalloc[s + 1]) * dev_out_elems(c->layers, w->last, B()),
                              esz);
            w->bytes_sent += (uint64_t)dev_out_elems(c->layers, w->last, B()) * esz;
        }
        const long lrows = rows_of(layer(w->last), B());
        const int32_t *labels = (s + 1 == n()) ? w->labels + (long)(t % c->n_data) * lrows : nullptr;
        cudaEvent_t last_l0 = nullptr;
        auto body = [&](float *loss_dst) {
        if (w->fbias && w->n_breg)  // vertical sync, bf16: fp32 biases of the stashed version `slot`
            CK(regions_bf16_to_f32(static_cast<const __nv_bfloat16 *>(w->wslot[slot]), w->fbias, w->breg_off,
                                   w->breg_cnt, w->n_breg, w->stream));
        for (int l = w->first; l <= w->last; ++l) {
            const pd_layer_desc &d = layer(l);
            const void *x = layer_input(l, t, j);
            void *y = l < w->last ? elem_ptr(w->act[l + 1 - w->first],
                                             (long)(j % w->k) * dev_in_elems(c->layers, l + 1, B()), esz)
                                  : y_last;
            if (const int run = lstm_wave_run(l)) {
                lstm_wave_forward(l, run, t, j, slot, y_last);
                l += run - 1;
                continue;
            }
            cudaEvent_t l0 = lstart();
            cudaEvent_t k0 = kstart(0);
            if (d.kind == PD_LINEAR) {
                LayerCtx lc{c, w, bf16};
                // the previous kernel on the stream is the previous layer's GEMM: this one may
                // start early and prefetch its weights (Gemm::pdl)
                const int pdl = bf16 && l > w->first && layer(l - 1).kind == PD_LINEAR && !w->fbias;
                linear_forward(lc, d, Wl(l, slot), bias_f32(l, slot), x, y, w->ws, w->ws_bytes, pdl);
            } else if (d.kind == PD_LSTM) {
                lstm_forward(l, j, slot, x, y);
            } else if (d.kind == PD_EMBEDDING) {
                CK(embedding_fwd(bf16, static_cast<const int32_t *>(x), Wl(l, slot), y, rows_of(d, B()), d.out,
                                 w->stream));
            } else if (d.kind == PD_CONV3X3) {
                conv_forward(l, slot, x, y);
            } else if (d.kind == PD_MAXPOOL2) {
                const bool outpad = l + 1 < (int)c->layers.size() && padded_in(layer(l + 1));
                CK(pool_fwd(bf16, x, y, B(), d.height, d.width, d.in, outpad, w->stream));
            } else {
                throw CudaFail{cudaErrorNotSupported, "layer kind not implemented"};
            }
            kend(0, k0);
            if (l < w->last || s + 1 < n()) lend(l, 'F', l0);
            else last_l0 = l0;  // the loss belongs to the model's last layer
        }
        if (s + 1 == n()) {
            if (loss_dst == w->loss_scratch) CK(cudaMemsetAsync(loss_dst, 0, 4, w->stream));
            cudaEvent_t k6 = kstart(6);
            CK(softmax_ce(w->logits, bf16, labels, lrows, layer(w->last).out, w->dlogits, loss_dst, w->stream));
            kend(6, k6);
            lend(w->last, 'F', last_l0);
        }
        };
        if (op_graphs_ok()) {
            const std::vector<uintptr_t> key = {0, (uintptr_t)slot, (uintptr_t)(j % w->k),
                                                (uintptr_t)layer_input(w->first, t, j), (uintptr_t)y_last,
                                                (uintptr_t)labels};
            opgraph_run(key, [&] { body(w->loss_scratch); });
            if (s + 1 == n())
                CK(cudaMemcpyAsync(w->losses + t, w->loss_scratch, 4, cudaMemcpyDeviceToDevice, w->stream));
        } else {
            body(w->losses + t);
        }
        if (s + 1 == n()) {
        } else {
            const int Rn = c->plan.stage[s + 1].replicas;
            Link &L = get_link(c, L_ACT, w->id, c->worker_id(s + 1, t % Rn));
            link_post(c, L, w->stream, w->vc);
        }
        record_end();
    }

    // message index of minibatch t on the act link (stage ps replica t%Rp) -> (ps+1 replica t%Rc)
    int64_t act_msg_index(int ps, int t) const {
        const int Rp = c->plan.stage[ps].replicas, Rc = c->plan.stage[ps + 1].replicas;
        int64_t cnt = 0;
        for (int u = 0; u < t; ++u)
            if (u % Rp == t % Rp && u % Rc == t % Rc) ++cnt;
        return cnt;
    }

    struct BwdCtx {
        bool fused;   // bf16 unreplicated: optimizer update fused into the dW GEMMs
        float *gdst;  // fp32 gradient buffer otherwise (gbuf or replica round buffer)
        int nslot;    // slot receiving the next version
        int sslot;    // stashed version's slot
    };

    // dX = G W (B(n,k) given by the caller) fused with the previous layer's ReLU derivative
    void gemm_dx(int l, int M, int N, int K, const void *G, long ldg, const void *W, long ldw, const void *x, void *dx) {
        const bool prev_relu = l > 0 && layer(l - 1).act == PD_ACT_RELU;
        Gemm g;
        g.M = M;
        g.N = N;
        g.K = K;
        g.A = G;
        g.lda = ldg;
        g.amaj = KMAJ;
        g.B = W;
        g.ldb = ldw;
        g.bmaj = MNMAJ;
        g.epi = prev_relu ? EPI_MASK : EPI_STORE;
        g.out = dx;
        g.ldo = N;
        g.mask = prev_relu ? x : nullptr;
        g.ldm = N;
        g.workspace = w->ws;
        g.workspace_bytes = w->ws_bytes;
        CK(run_gemm(bf16, g, w->stream));
    }

    // PD_DW_SPLIT_K: fused-path weight gradients with K >= this many rows (and M, N >= 256) run
    // as GEMM -> fp32 gradient -> update kernel instead of the fused-epilogue GEMM (0 = never).
    // Default 1024: GNMT-8 at N = 1 8.68k -> 9.74k samples/s (the LSTM W_ih / W_hh and
    // classifier gradients, K = T*B = 3200); the MLP's K = 256 dW stays fused
    bool split_dw(int M, int N, int K) const {
        const char *e = getenv("PD_DW_SPLIT_K");  // read per call (tests toggle it)
        const int kmin = e ? atoi(e) : 1024;
        return bf16 && kmin > 0 && K >= kmin && M >= 256 && N >= 256 && (long)M * N % 4 == 0;
    }

    // dW (M x N, row-major at parameter offset woff) = A^T B over K rows, either fused with
    // the optimizer update (writing the next version) or stored as an fp32 gradient
    void gemm_dw(const BwdCtx &bc, long woff, int M, int N, int K, const void *A, long lda, const void *Bm, long ldb) {
        Gemm g;
        g.M = M;
        g.N = N;
        g.K = K;
        g.A = A;
        g.lda = lda;
        g.amaj = MNMAJ;
        g.B = Bm;
        g.ldb = ldb;
        g.bmaj = MNMAJ;
        g.ldo = N;
        if (bc.fused && split_dw(M, N, K)) {
            // long-K weight gradients (LSTM W_ih / W_hh over T*B rows, classifier): the plain
            // 2-CTA GEMM into an fp32 gradient, then one vectorised update pass.  The fused
            // epilogue's single-CTA 128-wide tiles ingest 2x the operand bytes per FLOP
            const bool adam = c->cfg.optimizer == PD_ADAM;
            g.epi = EPI_F32;
            g.out = w->gbuf + woff;
            cudaEvent_t k0 = kstart(2);
            CK(run_gemm(bf16, g, w->stream));
            kend(2, k0);
            k0 = kstart(7);
            CK(update_from_grad(w->master + woff, static_cast<__nv_bfloat16 *>(elem_ptr(w->wslot[bc.nslot], woff, esz)),
                                w->gbuf + woff, (long)M * N, c->cfg.optimizer, adam ? w->adam_m + woff : nullptr,
                                adam ? w->adam_v + woff : nullptr, c->cfg.lr, c->cfg.beta1, c->cfg.beta2, c->cfg.eps,
                                w->updates_total + 1, w->stream));
            kend(7, k0);
            return;
        }
        if (bc.fused) {
            const bool adam = c->cfg.optimizer == PD_ADAM;
            g.epi = adam ? EPI_ADAM : EPI_SGD;
            g.master = w->master + woff;
            g.slot = elem_ptr(w->wslot[bc.nslot], woff, esz);
            g.adam_m = adam ? w->adam_m + woff : nullptr;
            g.adam_v = adam ? w->adam_v + woff : nullptr;
            g.lr = c->cfg.lr;
            g.b1 = c->cfg.beta1;
            g.b2 = c->cfg.beta2;
            g.eps = c->cfg.eps;
            g.step = w->updates_total + 1;
        } else {
            g.epi = EPI_F32;
            g.out = bc.gdst + woff;
        }
        cudaEvent_t k0 = kstart(2);
        CK(run_gemm(bf16, g, w->stream));
        kend(2, k0);
    }

    // bias gradient = column sums of G [rows][cols] (+ fused update)
    void bias_update(const BwdCtx &bc, long boff, const void *G, long rows, int cols) {
        if (bc.fused)
            CK(bias_grad(G, bf16, rows, cols, nullptr, w->master + boff,
                         static_cast<__nv_bfloat16 *>(elem_ptr(w->wslot[bc.nslot], boff, esz)), c->cfg.optimizer,
                         w->adam_m ? w->adam_m + boff : nullptr, w->adam_v ? w->adam_v + boff : nullptr, c->cfg.lr,
                         c->cfg.beta1, c->cfg.beta2, c->cfg.eps, w->updates_total + 1, w->stream));
        else
            CK(bias_grad(G, bf16, rows, cols, bc.gdst + boff, nullptr, nullptr, 0, nullptr, nullptr, 0.f, 0.f, 0.f,
                         0.f, 1, w->stream));
    }

    // LSTM b_ih and b_hh receive the same gradient (sum over rows of da): on the fused path it is
    // reduced ONCE -- written to the gradient scratch while b_ih is updated -- and b_hh is updated
    // from the scratch by the vectorised update kernel
    void bias_update_pair(const BwdCtx &bc, long boff_ih, long boff_hh, const void *G, long rows, int cols) {
        if (!bc.fused) {
            bias_update(bc, boff_ih, G, rows, cols);
            bias_update(bc, boff_hh, G, rows, cols);
            return;
        }
        const bool adam = c->cfg.optimizer == PD_ADAM;
        CK(bias_grad(G, bf16, rows, cols, w->gbuf + boff_ih, w->master + boff_ih,
                     static_cast<__nv_bfloat16 *>(elem_ptr(w->wslot[bc.nslot], boff_ih, esz)), c->cfg.optimizer,
                     adam ? w->adam_m + boff_ih : nullptr, adam ? w->adam_v + boff_ih : nullptr, c->cfg.lr,
                     c->cfg.beta1, c->cfg.beta2, c->cfg.eps, w->updates_total + 1, w->stream));
        const cudaError_t e = update_from_grad(
            w->master + boff_hh, static_cast<__nv_bfloat16 *>(elem_ptr(w->wslot[bc.nslot], boff_hh, esz)),
            w->gbuf + boff_ih, cols, c->cfg.optimizer, adam ? w->adam_m + boff_hh : nullptr,
            adam ? w->adam_v + boff_hh : nullptr, c->cfg.lr, c->cfg.beta1, c->cfg.beta2, c->cfg.eps,
            w->updates_total + 1, w->stream);
        if (e == cudaErrorInvalidValue) bias_update(bc, boff_hh, G, rows, cols);  // unaligned: reduce again
        else CK(e);
    }

    void linear_backward(int l, const void *x, const void *G, void *dx, const BwdCtx &bc) {
        const pd_layer_desc &d = layer(l);
        const long rows = rows_of(d, B());
        if (dx) {
            cudaEvent_t k0 = kstart(1);
            gemm_dx(l, (int)rows, d.in, d.out, G, d.out, Wl(l, bc.sslot), d.in, x, dx);
            kend(1, k0);
        }
        gemm_dw(bc, c->poff[l], d.out, d.in, (int)rows, G, d.out, x, d.in);
        cudaEvent_t k0 = kstart(3);
        bias_update(bc, c->poff[l] + (long)d.out * d.in, G, rows, d.out);
        kend(3, k0);
    }

    // LSTM saved state of layer l for local index j
    struct LstmState {
        float *gates, *c;
        void *h;
    };
    LstmState lstm_state(int l, int j) const {
        const pd_layer_desc &d = layer(l);
        const long TB = (long)d.seq_len * B(), H = d.out;
        char *base = static_cast<char *>(w->aux[l - w->first]) + (long)(j % w->k) * w->aux_bytes[l - w->first];
        LstmState st;
        st.gates = reinterpret_cast<float *>(base);
        st.c = reinterpret_cast<float *>(base + align_up(TB * 4 * H * 4, 256));
        st.h = base + align_up(TB * 4 * H * 4, 256) + align_up(TB * H * 4, 256);
        return st;
    }
    // parameter offsets of W_ih, W_hh, b_ih, b_hh
    long lstm_off(int l, int which) const {
        const pd_layer_desc &d = layer(l);
        const long H = d.out, I = d.in;
        const long o[4] = {0, 4 * H * I, 4 * H * I + 4 * H * H, 4 * H * I + 4 * H * H + 4 * H};
        return c->poff[l] + o[which];
    }
    const float *param_f32(long off, int slot) const { return fwd_f32(off, slot); }

    // Run `body` (a sequence of launches on w->stream) through a cached CUDA graph.
    template <typename F>
    void graph_run(const std::tuple<int, int, int, int, const void *> &key, F body) {
        auto it = w->graphs.find(key);
        if (it == w->graphs.end()) {
            const uint64_t before = tl_launches;
            CK(cudaStreamBeginCapture(w->stream, cudaStreamCaptureModeRelaxed));
            try {
                body();
            } catch (...) {
                cudaGraph_t g;
                cudaStreamEndCapture(w->stream, &g);
                if (g) cudaGraphDestroy(g);
                throw;
            }
            cudaGraph_t g;
            CK(cudaStreamEndCapture(w->stream, &g));
            cudaGraphExec_t ex;
            CK(cudaGraphInstantiate(&ex, g, 0));
            CK(cudaGraphDestroy(g));
            const int nk = (int)(tl_launches - before);
            tl_launches = before;
            it = w->graphs.emplace(key, std::make_pair(ex, nk)).first;
        }
        CK(cudaGraphLaunch(it->second.first, w->stream));
        tl_launches += it->second.second;  // count the kernels the graph runs
    }

    template <typename F>
    void opgraph_run(const std::vector<uintptr_t> &key, F body) {
        auto it = w->opgraphs.find(key);
        if (it == w->opgraphs.end()) {
            const uint64_t before = tl_launches;
            capturing = true;
            CK(cudaStreamBeginCapture(w->stream, cudaStreamCaptureModeRelaxed));
            try {
                body();
            } catch (...) {
                cudaGraph_t g = nullptr;
                cudaStreamEndCapture(w->stream, &g);
                if (g) cudaGraphDestroy(g);
                capturing = false;
                throw;
            }
            cudaGraph_t g;
            CK(cudaStreamEndCapture(w->stream, &g));
            capturing = false;
            cudaGraphExec_t ex;
            CK(cudaGraphInstantiate(&ex, g, 0));
            CK(cudaGraphDestroy(g));
            const int nk = (int)(tl_launches - before);
            tl_launches = before;
            if (w->opgraphs.size() > 4096) {
                for (auto &kv : w->opgraphs) cudaGraphExecDestroy(kv.second.first);
                w->opgraphs.clear();
            }
            it = w->opgraphs.emplace(key, std::make_pair(ex, nk)).first;
        }
        CK(cudaGraphLaunch(it->second.first, w->stream));
        tl_launches += it->second.second;
    }

    // whole-op graphs: bf16 fused all-linear SGD stages (the launch-bound MLP path), and only
    // when no per-kernel timing is requested (event timing cannot live inside a graph)
    bool op_graphs_ok() const {
        if (!bf16 || c->cfg.optimizer != PD_SGD || c->layer_prof) return false;
        if (c->plan.stage[w->stage].replicas != 1) return false;
        if (timing && c->ktime_mask) return false;
        for (int l = w->first; l <= w->last; ++l)
            if (layer(l).kind != PD_LINEAR) return false;
        return true;
    }

    // Persistent recurrences (lstm_rec.cu): bf16 path, supported shape, co-resident grid, and
    // no other LSTM-bearing worker on this GPU (two spinning grids could each hold half the
    // SMs the other needs).  PD_LSTM_REC=0 forces the per-step path.
    bool use_lstm_rec(const pd_layer_desc &d, int Bn) { return lstm_rec_allowed() && lstm_rec_supported(Bn, d.out); }
    bool lstm_rec_allowed() {
        if (!bf16) return false;
        if (w->lstm_rec < 0) {
            const char *env = getenv("PD_LSTM_REC");
            int others = 0;
            for (auto &o : c->W) {
                if (!o || o.get() == w || o->device != w->device) continue;
                for (int l = o->first; l <= o->last; ++l)
                    if (c->layers[l].kind == PD_LSTM) {
                        ++others;
                        break;
                    }
            }
            w->lstm_rec = (env && env[0] == '0') || others ? 0 : 1;
        }
        return w->lstm_rec != 0;
    }

    // ---------------- wavefront over a run of LSTM layers (lstm_wave.cu)
    // Length of the run of LSTM layers starting at l that runs as one wavefront (>= 2 equal
    // layers, H = in = out, same T; bf16; the co-residency rule of use_lstm_rec), else 0.
    int lstm_wave_run(int l) {
        const char *env = getenv("PD_LSTM_WAVE");  // 0 = per-layer recurrences (tools / tests)
        if ((env && env[0] == '0') || !bf16 || c->layer_prof) return 0;
        const pd_layer_desc &d = layer(l);
        if (d.kind != PD_LSTM || d.in != d.out || !lstm_rec_allowed()) return 0;
        // a chain of equal LSTMs is cut into runs of at most G layers (PD_LSTM_WAVE_L; default
        // the kernel's maximum).  Measured on GNMT-8 / -16: the wave time is set by
        // per-wave latency, not by the weight bytes, so fewer, longer runs win (G = 2: 3.8k /
        // 2.0k samples/s, G = 8: 8.1k / 4.7k, G = 16: - / 5.3k) even though 4 layers' weights
        // would stay L2-resident
        const char *ge = getenv("PD_LSTM_WAVE_L");
        int G = ge ? atoi(ge) : LSTM_WAVE_MAX_L;
        G = std::max(2, std::min(G, LSTM_WAVE_MAX_L));
        int cs = l;
        while (cs > w->first && lstm_chain(cs - 1)) --cs;
        if ((l - cs) % G) return 0;  // not the start of a run
        int n = 1;
        while (n < G && lstm_chain(l + n - 1)) ++n;
        if (n < 2 || !lstm_wave_supported(n, B(), d.out, d.in)) return 0;
        return n;
    }
    // the run (start, length) containing layer l, or length 0
    int lstm_wave_run_of(int l, int &start) {
        int cs = l;
        while (cs > w->first && lstm_chain(cs - 1)) --cs;
        for (int s0 = cs; s0 <= l;) {
            const int n = lstm_wave_run(s0);
            if (n == 0) return 0;
            if (l < s0 + n) {
                start = s0;
                return n;
            }
            s0 += n;
        }
        return 0;
    }
    // layers a and a+1 are equal square LSTMs (a wavefront run continues through them)
    bool lstm_chain(int a) const {
        if (a + 1 > w->last) return false;
        const pd_layer_desc &p = layer(a), &q = layer(a + 1);
        return p.kind == PD_LSTM && q.kind == PD_LSTM && p.in == p.out && q.in == p.out && q.out == p.out &&
               q.seq_len == p.seq_len;
    }

    void lstm_wave_forward(int l0, int L, int t, int j, int slot, void *y_last) {
        const pd_layer_desc &d = layer(l0);
        const int T = d.seq_len, Bn = B(), H = d.out;
        LstmWaveDesc wd;
        wd.bwd = 0, wd.L = L, wd.T = T, wd.B = Bn, wd.H = H;
        wd.x = static_cast<const __nv_bfloat16 *>(layer_input(l0, t, j));
        wd.cnt = w->lstm_cnt;
        // the run's inner layers read their input straight from the previous layer's saved h
        // (layer_input); the top layer's epilogue also stores h into the next layer's input
        // stash or the stage output -- the consumer's receive slot, over NVLink when the
        // consumer is another GPU -- so no copy follows the kernel
        const int top = l0 + L - 1;
        wd.h_out = static_cast<__nv_bfloat16 *>(
            top < w->last ? elem_ptr(w->act[top + 1 - w->first], (long)(j % w->k) * dev_in_elems(c->layers, top + 1, B()),
                                     esz)
                          : y_last);
        for (int i = 0; i < L; ++i) {
            const int l = l0 + i;
            LstmState st = lstm_state(l, j);
            wd.W_ih[i] = static_cast<const __nv_bfloat16 *>(elem_ptr(w->wslot[slot], lstm_off(l, 0), esz));
            wd.W_hh[i] = static_cast<const __nv_bfloat16 *>(elem_ptr(w->wslot[slot], lstm_off(l, 1), esz));
            wd.b_ih[i] = param_f32(lstm_off(l, 2), slot);
            wd.b_hh[i] = param_f32(lstm_off(l, 3), slot);
            wd.gates[i] = st.gates, wd.c[i] = st.c, wd.h[i] = static_cast<__nv_bfloat16 *>(st.h);
        }
        cudaEvent_t k0 = kstart(4);
        CK(lstm_wave(wd, w->stream));
        kend(4, k0);
    }

    // Backward wave of a short run (<= 3 layers: the wave leaves >= 52 SMs idle) with the run's
    // weight gradients computed WHILE the wave runs, on the idle SMs: the W_ih / W_hh GEMMs of
    // every layer (6 streams) split K = T*B into chunks of timesteps, run the chunks last
    // timesteps first, and wait per chunk for the wave's step counter of that layer (the wave
    // finishes timesteps in descending order), reduce-adding fp32 partials into the zeroed
    // gradient; the optimizer updates follow the wave.  The GEMM streams launch only once
    // every CTA of the wave is resident (a stream wait on the wave's start counter), so they
    // can never take SMs the spinning wave needs.  Only for a worker alone on its GPU.
    // Returns false (nothing issued) when not applicable.
    bool wave_dw_overlap(int l0, int L, int t, int j, LstmWaveDesc &wd, void *dx, const BwdCtx &bc) {
        if (!bc.fused || L > 3 || !w->dw_stream[0]) return false;
        if (const char *e = getenv("PD_WAVE_DW")) {  // 0: weight gradients after the wave (tests)
            if (atoi(e) == 0) return false;
        }
        for (auto &o : c->W)
            if (o && o.get() != w && o->device == w->device) return false;
        cudaStreamCaptureStatus cap_st = cudaStreamCaptureStatusNone;  // (the host gate cannot be captured)
        CK(cudaStreamIsCapturing(w->stream, &cap_st));
        if (cap_st != cudaStreamCaptureStatusNone) return false;
        const int T = wd.T, Bn = wd.B, H = wd.H;
        int wcl = 0;
        const int wgrid = lstm_wave_grid(true, L, H, &wcl);
        int sms = 0;
        CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, w->device));
        const int ng = 2 * L;
        const int cap = (sms - wgrid) / ng / 2 * 2;  // CTAs per GEMM (pairs)
        if (cap < 4) return false;
        const long TB = (long)T * Bn;
        unsigned *flag_dev = nullptr;
        CK(cudaHostGetDevicePointer(reinterpret_cast<void **>(&flag_dev), w->wave_flag, 0));
        // zeroed gradients (reduce-add targets), then the wave; the gradient GEMMs are launched
        // only once the host sees every wave CTA resident (a device-side gate could let them
        // take the SMs the wave's clusters need first)
        for (int i = 0; i < L; ++i)
            for (int m = 0; m < 2; ++m)
                CK(cudaMemsetAsync(w->gbuf + lstm_off(l0 + i, m), 0, (size_t)4 * H * H * 4, w->stream));
        CK(cudaEventRecord(w->ev_fork, w->stream));
        wd.started = w->lstm_cnt + LSTM_WAVE_MAX_L;
        wd.started_host = flag_dev;
        wd.epoch = ++w->wave_epoch;
        cudaEvent_t k0 = kstart(5);
        CK(lstm_wave(wd, w->stream));
        kend(5, k0);
        {
            const auto t0 = std::chrono::steady_clock::now();
            while (*reinterpret_cast<volatile unsigned *>(w->wave_flag) != wd.epoch) {
                if (c->abort) throw Abort{};
                if (std::chrono::steady_clock::now() - t0 > std::chrono::seconds(20))
                    throw CudaFail{cudaErrorLaunchTimeout, "backward wave never became resident"};
                std::this_thread::yield();
            }
        }
        const int chunk_steps = 10;  // availability granularity (the chunk's K = 10 * B rows)
        // the new version goes to another slot than the one the wave reads (k_s >= 2): each
        // matrix's optimizer update can follow its gradient GEMM on the same stream, under the
        // wave; with k_s = 1 (in place) the updates wait for the wave and the bottom layer's dX
        const bool early = bc.nslot != bc.sslot;
        const bool adam = c->cfg.optimizer == PD_ADAM;
        int g = 0;
        for (int i = L - 1; i >= 0; --i)
            for (int m = 0; m < 2; ++m, ++g) {
                const int l = l0 + i;
                cudaStream_t st = w->dw_stream[g];
                CK(cudaStreamWaitEvent(st, w->ev_fork, 0));
                const int steps = m == 0 ? T : T - 1;  // W_hh pairs da[t+1] with h[t]
                Gemm gg;
                gg.M = 4 * H;
                gg.N = H;
                gg.K = (int)((long)steps * Bn);
                gg.A = m == 0 ? static_cast<const void *>(wd.da[i]) : elem_ptr(wd.da[i], (long)Bn * 4 * H, esz);
                gg.lda = 4 * H;
                gg.amaj = MNMAJ;
                gg.B = m == 0 ? layer_input(l, t, j) : lstm_state(l, j).h;
                gg.ldb = H;
                gg.bmaj = MNMAJ;
                gg.epi = EPI_F32;
                gg.atomic_out = 1;
                gg.ksplit = (steps + chunk_steps - 1) / chunk_steps;
                gg.out = w->gbuf + lstm_off(l, m);
                gg.ldo = H;
                gg.max_ctas = cap;
                gg.wait_cnt = w->lstm_cnt + i;
                gg.wait_T = steps;  // row r of A is step r / B (+1 for W_hh), done at cnt >= (T - step) * per
                gg.wait_B = Bn;
                gg.wait_per = (unsigned)(H / 128) * (unsigned)wcl;
                CK(run_gemm(1, gg, st));
                if (early) {  // this matrix's update right behind its gradient (still under the wave)
                    const long woff = lstm_off(l, m);
                    CK(update_from_grad(w->master + woff,
                                        static_cast<__nv_bfloat16 *>(elem_ptr(w->wslot[bc.nslot], woff, esz)),
                                        w->gbuf + woff, 4L * H * H, c->cfg.optimizer, adam ? w->adam_m + woff : nullptr,
                                        adam ? w->adam_v + woff : nullptr, c->cfg.lr, c->cfg.beta1, c->cfg.beta2,
                                        c->cfg.eps, w->updates_total + 1, st));
                }
                CK(cudaEventRecord(w->dw_ev[g], st));
            }
        // the bottom layer's input gradient, then (after every gradient GEMM) the updates: with
        // k_s = 1 the W_ih update is in place and dX reads W_ih
        k0 = kstart(1);
        if (dx) gemm_dx(l0, (int)TB, H, 4 * H, wd.da[0], 4 * H, wd.W_ih[0], H, layer_input(l0, t, j), dx);
        kend(1, k0);
        for (int i = L - 1; i >= 0; --i) {  // biases: sums over the whole da, after the wave
            k0 = kstart(3);
            bias_update_pair(bc, lstm_off(l0 + i, 2), lstm_off(l0 + i, 3), wd.da[i], TB, 4 * H);
            kend(3, k0);
        }
        for (int k = 0; k < ng; ++k) CK(cudaStreamWaitEvent(w->stream, w->dw_ev[k], 0));
        if (!early)
            for (int i = L - 1; i >= 0; --i)
                for (int m = 0; m < 2; ++m) {
                    const long woff = lstm_off(l0 + i, m);
                    k0 = kstart(7);
                    CK(update_from_grad(w->master + woff,
                                        static_cast<__nv_bfloat16 *>(elem_ptr(w->wslot[bc.nslot], woff, esz)),
                                        w->gbuf + woff, 4L * H * H, c->cfg.optimizer, adam ? w->adam_m + woff : nullptr,
                                        adam ? w->adam_v + woff : nullptr, c->cfg.lr, c->cfg.beta1, c->cfg.beta2,
                                        c->cfg.eps, w->updates_total + 1, w->stream));
                    kend(7, k0);
                }
        return true;
    }

    void lstm_wave_backward(int l0, int L, int t, int j, const void *G, void *dx, const BwdCtx &bc) {
        const pd_layer_desc &d = layer(l0);
        const int T = d.seq_len, Bn = B(), H = d.out;
        const long TB = (long)T * Bn;
        if (!w->lstm_wda || L > w->lstm_wmax)  // sized in pd_stage_init: no allocation while others capture
            throw CudaFail{cudaErrorInvalidValue, "wavefront scratch not allocated"};
        LstmWaveDesc wd;
        wd.bwd = 1, wd.L = L, wd.T = T, wd.B = Bn, wd.H = H;
        wd.dy_top = static_cast<const __nv_bfloat16 *>(G);
        wd.cnt = w->lstm_cnt;
        for (int i = 0; i < L; ++i) {
            const int l = l0 + i;
            LstmState st = lstm_state(l, j);
            wd.W_ih[i] = static_cast<const __nv_bfloat16 *>(elem_ptr(w->wslot[bc.sslot], lstm_off(l, 0), esz));
            wd.W_hh[i] = static_cast<const __nv_bfloat16 *>(elem_ptr(w->wslot[bc.sslot], lstm_off(l, 1), esz));
            wd.gates[i] = st.gates, wd.c[i] = st.c;
            wd.da[i] = static_cast<__nv_bfloat16 *>(elem_ptr(w->lstm_wda, (long)i * TB * 4 * H, esz));
            wd.dc[i] = w->lstm_wdc + (long)i * Bn * H;
        }
        if (wave_dw_overlap(l0, L, t, j, wd, dx, bc)) return;
        cudaEvent_t k0 = kstart(5);
        CK(lstm_wave(wd, w->stream));
        kend(5, k0);
        // The bottom layer's input gradient (inner layers' are folded into the wavefront) and the
        // run's weight gradients + updates are independent GEMMs: the odd layers' go to the side
        // stream so two GEMMs share the machine (one M = 4H, N = H GEMM fills ~86 % of the CTA
        // pairs); the bottom layer's stay behind dX on the main stream, because with k_s = 1
        // its W_ih update is in place and dX reads W_ih
        CK(cudaEventRecord(w->ev_fork, w->stream));
        CK(cudaStreamWaitEvent(w->side, w->ev_fork, 0));
        k0 = kstart(1);
        if (dx) gemm_dx(l0, (int)TB, H, 4 * H, wd.da[0], 4 * H, wd.W_ih[0], H, layer_input(l0, t, j), dx);
        kend(1, k0);
        const cudaStream_t main = w->stream;
        for (int i = L - 1; i >= 0; --i) {
            const int l = l0 + i;
            if (i & 1) w->stream = w->side;
            gemm_dw(bc, lstm_off(l, 0), 4 * H, H, (int)TB, wd.da[i], 4 * H, layer_input(l, t, j), H);
            gemm_dw(bc, lstm_off(l, 1), 4 * H, H, (int)((T - 1) * (long)Bn), elem_ptr(wd.da[i], (long)Bn * 4 * H, esz),
                    4 * H, lstm_state(l, j).h, H);
            k0 = kstart(3);
            bias_update_pair(bc, lstm_off(l, 2), lstm_off(l, 3), wd.da[i], TB, 4 * H);
            kend(3, k0);
            w->stream = main;
        }
        CK(cudaEventRecord(w->ev_dw[0], w->side));
        CK(cudaStreamWaitEvent(w->stream, w->ev_dw[0], 0));
    }

    void lstm_forward(int l, int j, int slot, const void *x, void *y) {
        const pd_layer_desc &d = layer(l);
        const int T = d.seq_len, Bn = B(), H = d.out, I = d.in;
        const long TB = (long)T * Bn;
        LstmState st = lstm_state(l, j);
        // Gx = X W_ih^T for all T*B rows at once
        Gemm g;
        g.M = (int)TB;
        g.N = 4 * H;
        g.K = I;
        g.A = x;
        g.lda = I;
        g.B = elem_ptr(w->wslot[slot], lstm_off(l, 0), esz);
        g.ldb = I;
        g.epi = EPI_F32;
        g.out = w->lstm_gx;
        g.ldo = 4 * H;
        CK(run_gemm(bf16, g, w->stream));
        const float *bih = param_f32(lstm_off(l, 2), slot), *bhh = param_f32(lstm_off(l, 3), slot);
        if (use_lstm_rec(d, Bn)) {
            // all T steps in one persistent launch (lstm_rec.cu)
            CK(cudaMemsetAsync(w->lstm_cnt, 0, 1024 * sizeof(unsigned), w->stream));
            CK(lstm_rec_fwd(w->lstm_gx, bih, bhh,
                            static_cast<const __nv_bfloat16 *>(elem_ptr(w->wslot[slot], lstm_off(l, 1), esz)),
                            st.gates, st.c, static_cast<__nv_bfloat16 *>(st.h), w->lstm_cnt, T, Bn, H, w->stream));
            CK(cudaMemcpyAsync(y, st.h, (size_t)TB * H * esz, cudaMemcpyDeviceToDevice, w->stream));
            return;
        }
        // the recurrence writes h into the saved state only; one copy forwards it to y
        // (possibly another GPU's receive ring) so the captured graph is independent of y
        graph_run(std::make_tuple(l, 0, j % w->k, slot, (const void *)nullptr), [&] {
        for (int t = 0; t < T; ++t) {
            if (t > 0) {
                Gemm r;
                r.M = Bn;
                r.N = 4 * H;
                r.K = H;
                r.A = elem_ptr(st.h, (long)(t - 1) * Bn * H, esz);
                r.lda = H;
                r.B = elem_ptr(w->wslot[slot], lstm_off(l, 1), esz);
                r.ldb = H;
                r.epi = EPI_F32;
                r.out = w->lstm_gh;
                r.ldo = 4 * H;
                if (bf16) {  // M = B is tiny: split K across the machine, fp32 atomics
                    CK(cudaMemsetAsync(w->lstm_gh, 0, (size_t)Bn * 4 * H * 4, w->stream));
                    r.atomic_out = 1;
                    r.ksplit = 0;
                }
                CK(run_gemm(bf16, r, w->stream));
            }
            CK(lstm_cell_fwd(bf16, w->lstm_gx + (long)t * Bn * 4 * H, t > 0 ? w->lstm_gh : nullptr, bih, bhh,
                             t > 0 ? st.c + (long)(t - 1) * Bn * H : nullptr, st.gates + (long)t * Bn * 4 * H,
                             st.c + (long)t * Bn * H, elem_ptr(st.h, (long)t * Bn * H, esz), nullptr, Bn, H,
                             w->stream));
        }
        });
        CK(cudaMemcpyAsync(y, st.h, (size_t)TB * H * esz, cudaMemcpyDeviceToDevice, w->stream));
    }

    void lstm_backward(int l, int j, const void *x, const void *G, void *dx, const BwdCtx &bc) {
        const pd_layer_desc &d = layer(l);
        const int T = d.seq_len, Bn = B(), H = d.out, I = d.in;
        const long TB = (long)T * Bn;
        LstmState st = lstm_state(l, j);
        const void *Wih = elem_ptr(w->wslot[bc.sslot], lstm_off(l, 0), esz);
        const void *Whh = elem_ptr(w->wslot[bc.sslot], lstm_off(l, 1), esz);
        cudaEvent_t k0 = kstart(1);
        if (use_lstm_rec(d, Bn)) {
            CK(cudaMemsetAsync(w->lstm_cnt, 0, 1024 * sizeof(unsigned), w->stream));
            CK(lstm_rec_bwd(static_cast<const __nv_bfloat16 *>(G), st.gates, st.c,
                            static_cast<const __nv_bfloat16 *>(Whh), static_cast<__nv_bfloat16 *>(w->lstm_da),
                            w->lstm_cnt, T, Bn, H, w->stream));
        } else
        graph_run(std::make_tuple(l, 1, j % w->k, bc.sslot, G), [&] {
        CK(cudaMemsetAsync(w->lstm_dc, 0, (size_t)Bn * H * 4, w->stream));
        for (int t = T - 1; t >= 0; --t) {
            if (t < T - 1) {
                // dh_rec = da_{t+1} W_hh
                Gemm r;
                r.M = Bn;
                r.N = H;
                r.K = 4 * H;
                r.A = elem_ptr(w->lstm_da, (long)(t + 1) * Bn * 4 * H, esz);
                r.lda = 4 * H;
                r.amaj = KMAJ;
                r.B = Whh;
                r.ldb = H;
                r.bmaj = MNMAJ;
                r.epi = EPI_F32;
                r.out = w->lstm_dh;
                r.ldo = H;
                if (bf16) {  // M = B, N = H, K = 4H: split K, fp32 atomics
                    CK(cudaMemsetAsync(w->lstm_dh, 0, (size_t)Bn * H * 4, w->stream));
                    r.atomic_out = 1;
                    r.ksplit = 0;
                }
                CK(run_gemm(bf16, r, w->stream));
            }
            CK(lstm_cell_bwd(bf16, elem_ptr(G, (long)t * Bn * H, esz), t < T - 1 ? w->lstm_dh : nullptr,
                             st.gates + (long)t * Bn * 4 * H, st.c + (long)t * Bn * H,
                             t > 0 ? st.c + (long)(t - 1) * Bn * H : nullptr, w->lstm_dc,
                             elem_ptr(w->lstm_da, (long)t * Bn * 4 * H, esz), Bn, H, w->stream));
        }
        });
        if (dx) gemm_dx(l, (int)TB, I, 4 * H, w->lstm_da, 4 * H, Wih, I, x, dx);
        kend(1, k0);
        gemm_dw(bc, lstm_off(l, 0), 4 * H, I, (int)TB, w->lstm_da, 4 * H, x, I);
        gemm_dw(bc, lstm_off(l, 1), 4 * H, H, (int)((T - 1) * (long)Bn), elem_ptr(w->lstm_da, (long)Bn * 4 * H, esz),
                4 * H, st.h, H);
        k0 = kstart(3);
        bias_update_pair(bc, lstm_off(l, 2), lstm_off(l, 3), w->lstm_da, TB, 4 * H);
        kend(3, k0);
    }

    // ---------------- 3x3 convolution as an implicit GEMM on the padded grid
    ConvGeom conv_geom(const pd_layer_desc &d, int sign) const {
        ConvGeom g;
        const int Wp = d.width + 2;
        g.taps = 9;
        for (int tap = 0; tap < 9; ++tap) g.a_shift[tap] = sign * (((tap / 3) - 1) * Wp + (tap % 3) - 1);
        g.Hp = d.height + 2;
        g.Wp = Wp;
        return g;
    }

    void conv_forward(int l, int slot, const void *x, void *y) {
        const pd_layer_desc &d = layer(l);
        const int Cp = cpad8(d.in), Co = d.out, Hp = d.height + 2, Wp = d.width + 2;
        const long M = (long)B() * Hp * Wp;
        const long boff = c->poff[l] + (long)Co * 9 * Cp;
        if (!bf16) {
            const float *Wd = static_cast<const float *>(w->wslot[slot]) + c->poff[l];
            CK(conv_fwd_f32(static_cast<const float *>(x), Wd, Wd + (long)Co * 9 * Cp, static_cast<float *>(y), B(),
                            d.height, d.width, Cp, Co, d.act == PD_ACT_RELU, w->stream));
            return;
        }
        Gemm g;
        g.conv = conv_geom(d, +1);
        if (Cp == 8 && Co <= 64) {
            // RGB first layer: 9 taps x 8 channels packed into one K = 80 block
            g.conv.c8 = 1;
            g.M = (int)M;
            g.N = Co;
            g.K = 72;
            g.A = x;
            g.lda = 8;
            g.B = Wl(l, slot);
            g.ldb = 72;
            g.epi = EPI_STORE;
            g.out = y;
            g.ldo = Co;
            g.bias = fwd_f32(boff, slot);
            g.relu = d.act == PD_ACT_RELU;
            CK(run_gemm(1, g, w->stream));
            return;
        }
        g.conv.kpt = (Cp + 63) / 64;
        g.conv.b_koff = Cp;
        g.conv.a_inner = Cp;
        g.conv.b_inner = 9 * Cp;
        g.M = (int)M;
        g.N = Co;
        g.K = 9 * g.conv.kpt * 64;
        g.A = x;
        g.lda = Cp;
        g.B = Wl(l, slot);
        g.ldb = 9L * Cp;
        g.epi = EPI_STORE;
        g.out = y;
        g.ldo = Co;
        g.bias = fwd_f32(boff, slot);
        g.relu = d.act == PD_ACT_RELU;
        CK(run_gemm(1, g, w->stream));
    }

    void conv_backward(int l, const void *x, const void *G, void *dx, const BwdCtx &bc) {
        const pd_layer_desc &d = layer(l);
        const int Cp = cpad8(d.in), Co = d.out, Hp = d.height + 2, Wp = d.width + 2;
        const long M = (long)B() * Hp * Wp;
        const long n = c->pcount[l];
        const bool prev_relu = l > 0 && layer(l - 1).act == PD_ACT_RELU;
        float *gW = (bc.fused ? w->gbuf : bc.gdst) + c->poff[l];
        if (dx) {
            cudaEvent_t k0 = kstart(1);
            if (!bf16) {
                CK(conv_dx_f32(static_cast<const float *>(G),
                               static_cast<const float *>(w->wslot[bc.sslot]) + c->poff[l],
                               prev_relu ? static_cast<const float *>(x) : nullptr, static_cast<float *>(dx), B(),
                               d.height, d.width, Cp, Co, w->stream));
            } else {
                Gemm g;
                g.conv = conv_geom(d, -1);
                g.conv.kpt = (Co + 63) / 64;
                g.conv.b_noff = Cp;
                g.conv.a_inner = Co;
                g.conv.b_inner = 9 * Cp;
                g.M = (int)M;
                g.N = Cp;
                g.K = 9 * g.conv.kpt * 64;
                g.A = G;
                g.lda = Co;
                g.amaj = KMAJ;
                g.B = Wl(l, bc.sslot);
                g.ldb = 9L * Cp;
                g.bmaj = MNMAJ;
                g.epi = prev_relu ? EPI_MASK : EPI_STORE;
                g.mask = prev_relu ? x : nullptr;
                g.ldm = Cp;
                g.out = dx;
                g.ldo = Cp;
                CK(run_gemm(1, g, w->stream));
            }
            kend(1, k0);
        }
        cudaEvent_t k0 = kstart(2);
        CK(cudaMemsetAsync(gW, 0, (size_t)n * 4, w->stream));
        if (!bf16) {
            CK(conv_dw_f32(static_cast<const float *>(G), static_cast<const float *>(x), gW, B(), d.height, d.width,
                           Cp, Co, w->stream));
        } else if (Cp == 8) {
            // dW[co][tap*8 + ci] for all 9 taps of an 8-channel input in ONE GEMM (N = 72)
            Gemm g;
            g.M = Co;
            g.N = 72;
            g.K = (int)M;
            g.A = G;
            g.lda = Co;
            g.amaj = MNMAJ;
            g.B = x;
            g.ldb = 8;
            g.bmaj = MNMAJ;
            g.conv.c8 = 2;
            for (int tap = 0; tap < 9; ++tap) g.conv.a_shift[tap] = ((tap / 3) - 1) * Wp + (tap % 3) - 1;
            g.epi = EPI_F32;
            g.atomic_out = 1;
            g.out = gW;
            g.ldo = 72;
            CK(run_gemm(1, g, w->stream));
        } else if (Cp % 64 == 0) {
            // dW[co][tap*Cp + ci] for all 9 taps in ONE GEMM (N = 9*Cp): the dY tile is loaded
            // once per K-block for every tap of the tile instead of once per tap
            Gemm g;
            g.M = Co;
            g.N = 9 * Cp;
            g.K = (int)M;
            g.A = G;
            g.lda = Co;
            g.amaj = MNMAJ;
            g.B = x;
            g.ldb = Cp;
            g.bmaj = MNMAJ;
            g.conv.b_tapchunk = Cp;
            for (int tap = 0; tap < 9; ++tap) g.conv.a_shift[tap] = ((tap / 3) - 1) * Wp + (tap % 3) - 1;
            g.epi = EPI_F32;
            g.atomic_out = 1;
            g.ksplit = 0;
            g.out = gW;
            g.ldo = 9L * Cp;
            CK(run_gemm(1, g, w->stream));
        } else {
            const int Wpp = Wp;
            for (int tap = 0; tap < 9; ++tap) {
                // dW[:, tap, :] = dY^T X_shifted over every padded-grid pixel (halo rows are 0)
                Gemm g;
                g.M = Co;
                g.N = Cp;
                g.K = (int)M;
                g.A = G;
                g.lda = Co;
                g.amaj = MNMAJ;
                g.B = x;
                g.ldb = Cp;
                g.bmaj = MNMAJ;
                g.conv.b_kshift = ((tap / 3) - 1) * Wpp + (tap % 3) - 1;
                g.epi = EPI_F32;
                g.atomic_out = 1;
                g.ksplit = 0;  // auto
                g.out = gW + tap * Cp;
                g.ldo = 9L * Cp;
                CK(run_gemm(1, g, w->stream));
            }
        }
        CK(col_sum_tall(G, bf16, M, Co, gW + (long)Co * 9 * Cp, w->stream));
        if (bc.fused)
            CK(update_master(w->master + c->poff[l],
                             static_cast<__nv_bfloat16 *>(elem_ptr(w->wslot[bc.nslot], c->poff[l], esz)), nullptr,
                             w->self_grad_ptr, 1, c->poff[l], n, c->cfg.optimizer,
                             w->adam_m ? w->adam_m + c->poff[l] : nullptr, w->adam_v ? w->adam_v + c->poff[l] : nullptr,
                             c->cfg.lr, c->cfg.beta1, c->cfg.beta2, c->cfg.eps, w->updates_total + 1, w->stream));
        kend(2, k0);
    }

    void embedding_backward(int l, const void *tok, const void *G, const BwdCtx &bc) {
        const pd_layer_desc &d = layer(l);
        const long off = c->poff[l], n = (long)d.in * d.out;
        float *gE = bc.fused ? w->gbuf + off : bc.gdst + off;
        cudaEvent_t k0 = kstart(2);
        CK(cudaMemsetAsync(gE, 0, (size_t)n * 4, w->stream));
        CK(embedding_bwd(bf16, static_cast<const int32_t *>(tok), G, gE, rows_of(d, B()), d.out, w->stream));
        if (bc.fused) {
            // vectorised update (16-byte accesses); the generic replica kernel if unaligned
            const cudaError_t e = update_from_grad(
                w->master + off, static_cast<__nv_bfloat16 *>(elem_ptr(w->wslot[bc.nslot], off, esz)), gE, n,
                c->cfg.optimizer, w->adam_m ? w->adam_m + off : nullptr, w->adam_v ? w->adam_v + off : nullptr,
                c->cfg.lr, c->cfg.beta1, c->cfg.beta2, c->cfg.eps, w->updates_total + 1, w->stream);
            if (e == cudaErrorInvalidValue)
                CK(update_master(w->master + off, static_cast<__nv_bfloat16 *>(elem_ptr(w->wslot[bc.nslot], off, esz)),
                                 nullptr, w->self_grad_ptr, 1, off, n, c->cfg.optimizer,
                                 w->adam_m ? w->adam_m + off : nullptr, w->adam_v ? w->adam_v + off : nullptr,
                                 c->cfg.lr, c->cfg.beta1, c->cfg.beta2, c->cfg.eps, w->updates_total + 1, w->stream));
            else
                CK(e);
        }
        kend(2, k0);
    }

    // Backward of an all-linear stage on the bf16 fused path with the weight-gradient GEMM +
    // optimizer update of layer l (HBM-bound) on a side stream, overlapping the input-gradient
    // GEMM of layer l-1 (L2/latency-bound) on the main stream.  Hazards: dW_l rewrites W_l
    // (k_s = 1: in place) so it waits for dX_l; dX_{l-2} reuses dW_l's input buffer G_l, so it
    // waits for dW_l (3-deep rotation of the gradient scratch).
    void backward_linear_overlapped(int t, int j, const void *G_ext, const BwdCtx &bc, const void *dx_first) {
        const int s = w->stage;
        const int first = w->first, last = w->last;
        auto Gof = [&](int l) -> const void * {
            return l == last ? G_ext : w->scratch[(last - l - 1) % 3];
        };
#ifndef PD_FAULT_NO_DXWAIT
        // fork: the side stream's first dW reads G_ext (the gradient the main stream waited
        // for, or dlogits written by this worker's forward) -- also when no dX precedes it
        CK(cudaEventRecord(w->ev_fork, w->stream));
        CK(cudaStreamWaitEvent(w->side, w->ev_fork, 0));
#endif
        for (int l = last; l >= first; --l) {
            const pd_layer_desc &d = layer(l);
            const void *x = layer_input(l, t, j);
            const long rows = rows_of(d, B());
            const void *Gl = Gof(l);
            const bool need_dx = !(s == 0 && l == 0);
            if (need_dx) {
                void *dx;
                if (l == first) {
                    dx = const_cast<void *>(dx_first);
                } else {
                    dx = w->scratch[(last - l) % 3];
                    if (l + 2 <= last) CK(cudaStreamWaitEvent(w->stream, w->ev_dw[l + 2 - first], 0));
                }
                cudaEvent_t k0 = kstart(1);
                gemm_dx(l, (int)rows, d.in, d.out, Gl, d.out, Wl(l, bc.sslot), d.in, x, dx);
                kend(1, k0);
#ifndef PD_FAULT_NO_DXWAIT
                // dW_l + update rewrites W_l in place when k_s = 1: after dX_l has read it
                CK(cudaEventRecord(w->ev_dx[l - first], w->stream));
                CK(cudaStreamWaitEvent(w->side, w->ev_dx[l - first], 0));
#endif
            }
            // side stream: dW_l + fused update, bias
            cudaStream_t main = w->stream;
            w->stream = w->side;
            cudaEvent_t k0 = nullptr;
            if (split_dw(d.out, d.in, (int)rows)) {
                // long-K weight gradient (the classifier over T*B rows): 2-CTA GEMM -> fp32
                // gradient -> vectorised update (gemm_dw), not the single-CTA fused epilogue
                gemm_dw(bc, c->poff[l], d.out, d.in, (int)rows, Gl, d.out, x, d.in);
            } else {
                k0 = kstart(2);
                Gemm g;
                g.M = d.out;
                g.N = d.in;
                g.K = (int)rows;
                g.A = Gl;
                g.lda = d.out;
                g.amaj = MNMAJ;
                g.B = x;
                g.ldb = d.in;
                g.bmaj = MNMAJ;
                g.ldo = d.in;
                const bool adam = c->cfg.optimizer == PD_ADAM;
                const long woff = c->poff[l];
                g.epi = adam ? EPI_ADAM : EPI_SGD;
                g.master = w->master + woff;
                g.slot = elem_ptr(w->wslot[bc.nslot], woff, esz);
                g.adam_m = adam ? w->adam_m + woff : nullptr;
                g.adam_v = adam ? w->adam_v + woff : nullptr;
                g.lr = c->cfg.lr;
                g.b1 = c->cfg.beta1;
                g.b2 = c->cfg.beta2;
                g.eps = c->cfg.eps;
                g.step = w->updates_total + 1;
                CK(run_gemm(1, g, w->stream));
                kend(2, k0);
            }
            k0 = kstart(3);
            bias_update(bc, c->poff[l] + (long)d.out * d.in, Gl, rows, d.out);
            kend(3, k0);
            CK(cudaEventRecord(w->ev_dw[l - first], w->side));
            w->stream = main;
        }
        // join: everything of this backward is complete on the main stream
        CK(cudaStreamWaitEvent(w->stream, w->ev_dw[0], 0));
    }

    // ---------------- B(s, t)
    void backward(int t, int j) {
        const int s = w->stage;
        const int Rs = c->plan.stage[s].replicas;
        if (s + 1 < n()) {
            const int Rn = c->plan.stage[s + 1].replicas;
            Link &L = get_link(c, L_GRAD, c->worker_id(s + 1, t % Rn), w->id);
            link_wait(c, L, w->stream, act_msg_index(s, t), w->vc);
            hb_require(c->worker_id(s + 1, t % Rn), c->opB, t / Rn, "gradient used before its backward", t);
        }
        const int vst = w->fwd_version[j];
#ifdef PD_FAULT_STASH
        const int sslot = w->version % w->k;  // fault injection (tests): the latest, not the stashed, version
#else
        const int sslot = vst % w->k;  // stashed version (L1157-1161)
#endif
        if (s > 0) {
            const int Rp = c->plan.stage[s - 1].replicas;
            hb_require(c->worker_id(s - 1, t % Rp), c->opB, t / Rp - c->Galloc[s - 1],
                       "gradient receive slot rewritten before the backward that reads it", t);
        }
        trace('B', t, vst, vst);
        record_start();
        const int jr = j;  // round index on a replicated stage
        if (Rs > 1) {
            // gradient buffer parity jr%2 was last read by every replica in round jr-2 (rounds 0
            // and 1 of a run: by the previous run's last rounds -- wait for all of its messages)
            for (int r = 0; r < Rs; ++r) {
                if (r == w->replica) continue;
                Link &L = get_link(c, L_DONE, c->worker_id(s, r), w->id);
                link_wait(c, L, w->stream, jr >= 2 ? jr - 2 : -1, w->vc);
                hb_require(c->worker_id(s, r), c->opU, jr - 2,
                           "replica gradient buffer rewritten before the round that reads it", t);
            }
        }
        // gradient w.r.t. the stage output (pre-activation of the last layer)
        const void *G = (s + 1 == n()) ? w->dlogits
                                       : elem_ptr(w->gring, (long)(j % w->G) * dev_out_elems(c->layers, w->last, B()), esz);
        int cur = 0;
        // dW + optimizer update in one GEMM epilogue; GPipe: the weight gradient of the group's
        // i-th minibatch into its own fp32 buffer, aggregated by the group's update (L1277-1279)
        const bool fused = bf16 && Rs == 1 && !gpipe();
        float *gdst = Rs > 1 ? w->rgrad[jr & 1] : gpipe() ? w->gp_grad[t % k[0]] : w->gbuf;
        const int next_version = w->version + 1;
        const int nslot = next_version % w->k;
        if (!gpipe()) check_weight_slot(nslot, j, t);  // (GPipe: the group's update follows every B)
        BwdCtx bc{fused, gdst, nslot, sslot};
        bool all_linear = true;
        for (int l = w->first; l <= w->last; ++l) all_linear = all_linear && layer(l).kind == PD_LINEAR;
        if (fused && all_linear && !c->layer_prof) {
            const void *dx_first = nullptr;
            if (!(s == 0 && w->first == 0)) {
                const int Rp = c->plan.stage[s - 1].replicas;
                const int pw = c->worker_id(s - 1, t % Rp);
                dx_first = elem_ptr(c->shared[pw].grad,
                                    (long)((t / Rp) % c->Galloc[s - 1]) * dev_in_elems(c->layers, w->first, B()), esz);
                w->bytes_sent += (uint64_t)dev_in_elems(c->layers, w->first, B()) * esz;
            }
            if (op_graphs_ok()) {
                const std::vector<uintptr_t> key = {1, (uintptr_t)sslot, (uintptr_t)nslot, (uintptr_t)(j % w->k),
                                                    (uintptr_t)G, (uintptr_t)layer_input(w->first, t, j),
                                                    (uintptr_t)dx_first};
                opgraph_run(key, [&] { backward_linear_overlapped(t, j, G, bc, dx_first); });
            } else {
                backward_linear_overlapped(t, j, G, bc, dx_first);
            }
        } else
        for (int l = w->last; l >= w->first; --l) {
            // top layer of a wavefront run: the whole run's backward in one go
            int run_first = l;
            const int run = lstm_wave_run_of(l, run_first);
            const bool wave = run > 0 && run_first + run - 1 == l;
            if (wave) l = run_first;  // dX below is the run's bottom layer's
            const pd_layer_desc &d = layer(l);
            const void *x = layer_input(l, t, j);
            const bool need_dx = !(s == 0 && l == 0) && d.kind != PD_EMBEDDING;
            void *dx = nullptr;
            if (need_dx) {
                if (l == w->first) {
                    const int Rp = c->plan.stage[s - 1].replicas;
                    const int pw = c->worker_id(s - 1, t % Rp);
                    const int jp = t / Rp;
                    dx = elem_ptr(c->shared[pw].grad, (long)(jp % c->Galloc[s - 1]) * dev_in_elems(c->layers, l, B()), esz);
                    w->bytes_sent += (uint64_t)dev_in_elems(c->layers, l, B()) * esz;
                } else {
                    dx = w->scratch[cur ^ 1];
                }
            }
            cudaEvent_t l0 = lstart();
            if (wave) lstm_wave_backward(l, lstm_wave_run(l), t, j, G, dx, bc);
            else if (d.kind == PD_LINEAR) linear_backward(l, x, G, dx, bc);
            else if (d.kind == PD_LSTM) lstm_backward(l, j, x, G, dx, bc);
            else if (d.kind == PD_EMBEDDING) embedding_backward(l, x, G, bc);
            else if (d.kind == PD_CONV3X3) conv_backward(l, x, G, dx, bc);
            else if (d.kind == PD_MAXPOOL2) {
                if (dx) {
                    const bool dypad = l + 1 < (int)c->layers.size() && padded_in(layer(l + 1));
                    const bool prev_relu = l > 0 && layer(l - 1).act == PD_ACT_RELU;
                    cudaEvent_t k0 = kstart(1);
                    CK(pool_bwd(bf16, x, G, dx, B(), d.height, d.width, d.in, dypad, prev_relu, w->stream));
                    kend(1, k0);
                }
            } else throw CudaFail{cudaErrorNotSupported, "layer kind not implemented"};
            lend(l, 'B', l0);
            G = dx;
            cur ^= 1;
        }
        if (s > 0) {
            const int Rp = c->plan.stage[s - 1].replicas;
            Link &L = get_link(c, L_GRAD, w->id, c->worker_id(s - 1, t % Rp));
            link_post(c, L, w->stream, w->vc);
        }
        if (Rs > 1) {
            for (int r = 0; r < Rs; ++r) {
                if (r == w->replica) continue;
                Link &L = get_link(c, L_READY, w->id, c->worker_id(s, r));
                link_post(c, L, w->stream, w->vc);
            }
        }
        record_end();
    }

    // ---------------- U: weight update to the LATEST version (L1341-1353)
    void update(int t, int j) {
        const int s = w->stage;
        const int Rs = c->plan.stage[s].replicas;
        const int vin = w->version;
        const int nslot = (vin + 1) % w->k;
        trace('U', Rs > 1 || gpipe() ? j : t, vin, vin + 1);
        const bool adam = c->cfg.optimizer == PD_ADAM;
        const int step = w->updates_total + 1;
        if (Rs > 1) {
            // round j: reduce-scatter -> update -> all-gather through peer memory.  Every replica
            // waits for the others' gradients, reduces and updates its 1/R shard of the
            // parameters (sum in replica order, R7) and stores the new version of that shard
            // into every replica's next slot (and fp32 master); the round completes when every
            // replica has posted DONE -- the next forward reads the whole new version
            for (int r = 0; r < Rs; ++r) {
                if (r == w->replica) continue;
                Link &L = get_link(c, L_READY, c->worker_id(s, r), w->id);
                link_wait(c, L, w->stream, j, w->vc);
                hb_require(c->worker_id(s, r), c->opB, j, "replica gradient reduced before its backward", t);
            }
            auto shard_lo = [&](int r) { return (w->P * r / Rs) / 64 * 64; };
            const long lo = shard_lo(w->replica), hi = w->replica + 1 == Rs ? w->P : shard_lo(w->replica + 1);
            const float *w_in = bf16 ? w->master : static_cast<const float *>(w->wslot[vin % w->k]);
            CK(update_shard(w->rgrad_ptrs + (j & 1) * Rs, Rs, lo, hi, w_in, w->sync_f32 + (size_t)nslot * Rs,
                            bf16 ? w->sync_bf16 + (size_t)nslot * Rs : nullptr, Rs, c->cfg.optimizer, w->adam_m, w->adam_v,
                            c->cfg.lr, c->cfg.beta1, c->cfg.beta2, c->cfg.eps, step, w->stream));
            w->replica_bytes += (uint64_t)(Rs - 1) * (hi - lo) * (4 + 4 + (bf16 ? 2 : 0));
            for (int r = 0; r < Rs; ++r) {
                if (r == w->replica) continue;
                Link &L = get_link(c, L_DONE, w->id, c->worker_id(s, r));
                link_post(c, L, w->stream, w->vc);
            }
            for (int r = 0; r < Rs; ++r) {
                if (r == w->replica) continue;
                Link &L = get_link(c, L_DONE, c->worker_id(s, r), w->id);
                link_wait(c, L, w->stream, j, w->vc);
                hb_require(c->worker_id(s, r), c->opU, j, "new version used before every shard was written", t);
            }
        } else if (gpipe()) {
            // the flush: every backward of group j is done (stream order); mean of its D
            // gradients (t order, times 1/D) applied to the latest weights, new version into
            // slot nslot (the only other version alive is the one this group used)
            const float *w_in = bf16 ? w->master : static_cast<const float *>(w->wslot[vin % w->k]);
            CK(update_shard(w->gp_ptrs, k[0], 0, w->P, w_in, w->gp_out_f32 + nslot,
                            bf16 ? w->gp_out_bf16 + nslot : nullptr, 1, c->cfg.optimizer, w->adam_m, w->adam_v,
                            c->cfg.lr, c->cfg.beta1, c->cfg.beta2, c->cfg.eps, step, w->stream));
        } else if (!bf16) {
            const float *latest = static_cast<const float *>(w->wslot[vin % w->k]);
            float *next = static_cast<float *>(w->wslot[nslot]);
            if (adam)
                CK(adam_f32(latest, w->gbuf, next, w->adam_m, w->adam_v, w->P, c->cfg.lr, c->cfg.beta1, c->cfg.beta2,
                            c->cfg.eps, step, w->stream));
            else
                CK(sgd_f32(latest, w->gbuf, next, w->P, c->cfg.lr, w->stream));
        }
        // (bf16 unreplicated: the update was fused into B's dW epilogues)
        w->version = vin + 1;
        w->updates_total += 1;
        if (gpipe()) w->fwd_version.clear();  // every minibatch of the group is done
        else w->fwd_version.erase(j);
    }

    // PD_OP_TRACE=1: every op a worker issues, on stderr (diagnosing a stuck run)
    static bool op_trace() {
        static const bool v = getenv("PD_OP_TRACE") != nullptr;
        return v;
    }
    void run_ops() {
        const int Rs = c->plan.stage[w->stage].replicas;
        std::vector<Op> ops = gpipe() ? gpipe_ops(w->stage + 1 == n(), k[0], M) : worker_ops(Rs, w->replica, k[w->stage], M);
        w->run_base = w->version;
        w->vc.assign(c->nw, 0);
        // layers inside (not at the bottom of) an LSTM wavefront run: their input is the
        // previous layer's saved h (decided per run: it depends on the dtype, layer profiling
        // and the wavefront's co-residency rule)
        w->wave_inner.assign(w->last - w->first + 1, 0);
        for (int l = w->first; l <= w->last; ++l) {
            int st = l;
            if (lstm_wave_run_of(l, st) > 0 && st < l) w->wave_inner[l - w->first] = 1;
        }
        for (size_t i = 0; i < ops.size(); ++i) {
            const Op &op = ops[i];
            if (c->abort) throw Abort{};
            w->vc[w->id] = (int32_t)i + 1;  // a post during op i claims ops 0..i complete
            w->st_op = (int)i;
            if (op_trace()) fprintf(stderr, "[pd] worker %d op %zu %c t=%d j=%d v=%d\n", w->id, i, op.kind, op.t, op.j,
                                    w->version);
            if (op.kind == 'F') forward(op.t, op.j);
            else if (op.kind == 'B') backward(op.t, op.j);
            else update(op.t, op.j);
        }
    }
};

void worker_thread(pd_ctx *c, Worker *w, int M, std::vector<int> k) {
    tl_launches = 0;
    tl_worker = w;
    w->st_where = 0;
    try {
        CK(cudaSetDevice(w->device));
        Exec ex{c, w, M, k, c->cfg.dtype == PD_BF16, c->esz, c->cfg.record_trace >= 2};
        CK(cudaEventRecord(w->run_ev[0], w->stream));
        ex.run_ops();
        CK(cudaEventRecord(w->run_ev[1], w->stream));
        if (Exec::op_trace()) fprintf(stderr, "[pd] worker %d issued everything, synchronizing\n", w->id);
        w->st_where = 3;
        CK(cudaStreamSynchronize(w->stream));
        if (Exec::op_trace()) fprintf(stderr, "[pd] worker %d done\n", w->id);
    } catch (const CudaFail &f) {
        char buf[256];
        snprintf(buf, sizeof buf, "worker %d: %s failed: %s", w->id, f.what, cudaGetErrorString(f.e));
        c->fail(f.e == cudaErrorNotSupported ? PD_EUNSUPPORTED : PD_ECUDA, buf);
    } catch (const SlotViolation &v) {
        c->fail(PD_ESTATE, v.msg);
        if (w->stream) cudaStreamSynchronize(w->stream);
    } catch (const Abort &) {
        if (w->stream) cudaStreamSynchronize(w->stream);
    }
    w->launches = tl_launches;
    w->st_where = 4;
    tl_worker = nullptr;
    {
        std::lock_guard<std::mutex> g(c->done_mu);
        --c->running;
    }
    c->done_cv.notify_all();
}

}  // namespace

// ================================================================== C ABI
#define CHECK_CTX(ctx)                          \
    do {                                        \
        if (!(ctx)) return PD_EINVAL;           \
        if ((ctx)->sticky != PD_OK) return PD_ESTATE; \
    } while (0)

extern "C" {

const char *pd_strerror(pd_status s) {
    switch (s) {
    case PD_OK: return "ok";
    case PD_EINVAL: return "invalid argument";
    case PD_ENOMEM: return "out of memory";
    case PD_ECUDA: return "CUDA error";
    case PD_ENCCL: return "collective transport error";
    case PD_ESTATE: return "invalid state (earlier error or wrong call order)";
    case PD_EUNSUPPORTED: return "unsupported";
    case PD_EINFEASIBLE: return "no feasible plan";
    }
    return "unknown status";
}

const char *pd_last_error(pd_ctx *ctx) { return ctx ? ctx->err.c_str() : ""; }

pd_status pd_inflight(const pd_plan_t *plan, int noam, int *k_out) {
    if (!plan || !k_out || plan->num_stages < 1 || plan->num_stages > PD_MAX_STAGES) return PD_EINVAL;
    std::vector<int> k;
    pd_status st = inflight_counts(*plan, noam, k);
    if (st != PD_OK) return st;
    for (int s = 0; s < plan->num_stages; ++s) k_out[s] = k[s];
    return PD_OK;
}

pd_status pd_create(pd_ctx **out, const pd_plan_t *plan, const pd_layer_desc *layers, int num_layers,
                    const pd_train_cfg *cfg) {
    if (!out || !plan || !layers || !cfg || num_layers < 1) return PD_EINVAL;
    const int n = plan->num_stages;
    if (n < 1 || n > PD_MAX_STAGES) return PD_EINVAL;
    int expect = 0, total_workers = 0;
    for (int s = 0; s < n; ++s) {
        const pd_stage_desc &sd = plan->stage[s];
        if (sd.first_layer != expect || sd.last_layer < sd.first_layer || sd.replicas < 1) return PD_EINVAL;
        expect = sd.last_layer + 1;
        total_workers += sd.replicas;
    }
    if (expect != num_layers) return PD_EINVAL;
    if (cfg->minibatch < 1 || (cfg->dtype != PD_FP32 && cfg->dtype != PD_BF16)) return PD_EINVAL;
    if (cfg->optimizer != PD_SGD && cfg->optimizer != PD_ADAM) return PD_EINVAL;
    for (int l = 0; l < num_layers; ++l) {
        const pd_layer_desc &d = layers[l];
        if (d.in < 1 || d.out < 1 || numel_params(d) < 0) return PD_EINVAL;
        if (l > 0 && in_elems(d, 1) != out_elems(layers[l - 1], 1) && d.kind != PD_EMBEDDING) return PD_EINVAL;
        if (d.kind == PD_CONV3X3 || d.kind == PD_MAXPOOL2) {
            if (d.height < 2 || d.width < 2 || (d.kind == PD_MAXPOOL2 && ((d.height | d.width) & 1)))
                return PD_EINVAL;
            // a conv writes the padded layout: its consumer must be a conv or a pool
            if (d.kind == PD_CONV3X3 && (l + 1 >= num_layers || !padded_in(layers[l + 1]))) return PD_EUNSUPPORTED;
            if (cfg->dtype == PD_BF16 && d.kind == PD_MAXPOOL2 && d.in % 8) return PD_EUNSUPPORTED;
        }
        if (d.kind == PD_EMBEDDING && l != 0) return PD_EUNSUPPORTED;  // token ids enter at layer 0 only
        if (d.kind == PD_LSTM && d.seq_len < 2) return PD_EUNSUPPORTED;
        if (cfg->dtype == PD_BF16 && ((d.in % 8 && d.kind != PD_EMBEDDING && d.kind != PD_CONV3X3) || d.out % 8))
            return PD_EUNSUPPORTED;  // 16-byte rows for TMA
    }
    std::vector<int> kdef, kmax;
    if (inflight_counts(*plan, 0, kdef) != PD_OK) return PD_EINVAL;
    kmax = kdef;
    if (cfg->max_depth > 0) {
        if (inflight_counts(*plan, cfg->max_depth, kmax) != PD_OK) return PD_EINVAL;
        for (int s = 0; s < n; ++s) kmax[s] = std::max(kmax[s], kdef[s]);
    }
    // plan.noam is derived, not chosen: 0, or exactly k_0 = ceil(W / R_0) (L1021, R1)
    if (plan->noam != 0 && plan->noam != kdef[0]) return PD_EINVAL;
    if (cfg->sync_mode != PD_SYNC_STASH && cfg->sync_mode != PD_SYNC_VERTICAL && cfg->sync_mode != PD_SYNC_GPIPE)
        return PD_EINVAL;
    if (cfg->sync_mode != PD_SYNC_STASH)
        for (int s = 0; s < n; ++s)
            if (plan->stage[s].replicas != 1) return PD_EUNSUPPORTED;  // straight pipelines (§3.3, §5.4)
    // GPipe: every stage holds a whole flush group of D <= max(n, max_depth) minibatches (its
    // activation stash and receive rings); one weight version at a time (R27)
    if (cfg->sync_mode == PD_SYNC_GPIPE)
        for (int s = 0; s < n; ++s) kmax[s] = std::max({kmax[s], n, cfg->max_depth});
    pd_ctx *c = new pd_ctx;
    c->plan = *plan;
    c->layers.assign(layers, layers + num_layers);
    c->cfg = *cfg;
    c->n = n;
    c->nw = total_workers;
    c->kdef = kdef;
    c->kalloc = kmax;
    c->esz = cfg->dtype == PD_BF16 ? 2 : 4;
    int id = 0;
    for (int s = 0; s < n; ++s) {
        c->wbase.push_back(id);
        id += plan->stage[s].replicas;
    }
    c->Dalloc.assign(n, 0);
    c->Galloc.assign(n, 0);
    for (int s = 1; s < n; ++s) c->Dalloc[s] = recv_ring_depth(*plan, kmax, s);
#ifdef PD_FAULT_RECV_DEPTH
    for (int s = 1; s < n; ++s) c->Dalloc[s] = std::max(1, c->Dalloc[s] - 1);  // fault injection (tests)
#endif
    for (int s = 0; s + 1 < n; ++s) c->Galloc[s] = kmax[s];
    // vertical sync: stage s holds every version from the oldest tag still in flight to its
    // latest -- a window of k_0 versions at every stage (R25); rings sized as usual
    if (cfg->sync_mode == PD_SYNC_VERTICAL)
        for (int s = 0; s < n; ++s) c->kalloc[s] = kmax[0];
    c->poff.assign(num_layers, 0);
    c->pcount.assign(num_layers, 0);
    c->hcount.assign(num_layers, 0);
    for (int s = 0; s < n; ++s) {
        long off = 0;
        for (int l = plan->stage[s].first_layer; l <= plan->stage[s].last_layer; ++l) {
            c->poff[l] = off;
            c->hcount[l] = numel_params(layers[l]);
            c->pcount[l] = dev_params(layers[l]);
            off += align_up(c->pcount[l], 64);  // 256-byte aligned layer blocks
        }
    }
    c->W.resize(total_workers);
    c->shared.resize(total_workers);
    *out = c;
    return PD_OK;
}

pd_status pd_stage_init(pd_ctx *c, int stage, int replica, int dev, const float *const *init_params) {
    CHECK_CTX(c);
    if (stage < 0 || stage >= c->n || replica < 0 || replica >= c->plan.stage[stage].replicas) return PD_EINVAL;
    const int id = c->worker_id(stage, replica);
    if (c->W[id] || c->shared[id].valid) return PD_EINVAL;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
        cudaGetLastError();
        c->fail(PD_ECUDA, "no CUDA device");
        return PD_ECUDA;
    }
    if (dev < 0 || dev >= ndev) return PD_EINVAL;
    if (!driver()) {
        c->fail(PD_ECUDA, "CUDA driver entry points unavailable");
        return PD_ECUDA;
    }
    auto w = std::make_unique<Worker>();
    w->ctx = c;
    w->id = id;
    w->stage = stage;
    w->replica = replica;
    w->device = dev;
    w->first = c->plan.stage[stage].first_layer;
    w->last = c->plan.stage[stage].last_layer;
    w->k = c->kalloc[stage];
    w->D = stage > 0 ? c->Dalloc[stage] : 0;
    w->G = stage + 1 < c->n ? c->Galloc[stage] : 0;
    const int B = c->cfg.minibatch;
    const int esz = c->esz;
    const bool bf16 = c->cfg.dtype == PD_BF16;
    const int Rs = c->plan.stage[stage].replicas;
    try {
        CK(cudaSetDevice(dev));
        int major = 0;
        CK(cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev));
        if (major != 10) {
            c->fail(PD_EUNSUPPORTED, "requires an sm_100 (B200) device");
            return PD_EUNSUPPORTED;
        }
        CK(cudaStreamCreateWithFlags(&w->stream, cudaStreamNonBlocking));
        long P = 0;
        for (int l = w->first; l <= w->last; ++l) P = c->poff[l] + align_up(c->pcount[l], 64);
        w->P = P;
        // weights: stage buffer in the parameter layout, fp32 staging -> every slot
        float *stage_f32 = dalloc<float>(P * 4);
        std::vector<float> host(P, 0.f);
        for (int l = w->first; l <= w->last; ++l) {
            const float *src = init_params ? init_params[l - w->first] : nullptr;
            if (c->pcount[l] > 0) {
                if (!src) throw CudaFail{cudaErrorInvalidValue, "missing init params"};
                params_to_dev(c->layers[l], src, host.data() + c->poff[l]);
            }
        }
        CK(cudaMemcpy(stage_f32, host.data(), P * 4, cudaMemcpyHostToDevice));
        for (int q = 0; q < w->k; ++q) {
            void *slot = dalloc<void>(P * esz);
            if (bf16) CK(f32_to_bf16(stage_f32, static_cast<__nv_bfloat16 *>(slot), P, nullptr));
            else CK(cudaMemcpy(slot, stage_f32, P * 4, cudaMemcpyDeviceToDevice));
            w->wslot.push_back(slot);
        }
        if (bf16) w->master = stage_f32;
        else cudaFree(stage_f32);
        if (bf16 && c->cfg.sync_mode == PD_SYNC_VERTICAL) {
            std::vector<long> offs;
            std::vector<int> cnts;
            for (int l = w->first; l <= w->last; ++l) {
                const pd_layer_desc &d = c->layers[l];
                long o = -1, nb = 0;
                if (d.kind == PD_LINEAR) o = c->poff[l] + (long)d.out * d.in, nb = d.out;
                else if (d.kind == PD_CONV3X3) o = c->poff[l] + (long)d.out * 9 * cpad8(d.in), nb = d.out;
                else if (d.kind == PD_LSTM) o = c->poff[l] + 4L * d.out * d.in + 4L * d.out * d.out, nb = 8L * d.out;
                if (o >= 0) {
                    offs.push_back(o);
                    cnts.push_back((int)nb);
                }
            }
            w->n_breg = (int)offs.size();
            w->fbias = dalloc<float>(P * 4);
            if (w->n_breg) {
                w->breg_off = dalloc<long>(offs.size() * sizeof(long));
                w->breg_cnt = dalloc<int>(cnts.size() * sizeof(int));
                CK(cudaMemcpy(w->breg_off, offs.data(), offs.size() * sizeof(long), cudaMemcpyHostToDevice));
                CK(cudaMemcpy(w->breg_cnt, cnts.data(), cnts.size() * sizeof(int), cudaMemcpyHostToDevice));
            }
        }
        if (c->cfg.optimizer == PD_ADAM) {
            w->adam_m = dalloc<float>(P * 4);
            w->adam_v = dalloc<float>(P * 4);
        }
        w->gbuf = dalloc<float>(P * 4);
        {
            const float *one[1] = {w->gbuf};
            w->self_grad_ptr = dalloc<const float *>(sizeof(one));
            CK(cudaMemcpy(w->self_grad_ptr, one, sizeof(one), cudaMemcpyHostToDevice));
        }
        if (c->cfg.sync_mode == PD_SYNC_GPIPE) {
            // one fp32 gradient buffer per minibatch of the largest flush group
            for (int q = 0; q < w->k; ++q) w->gp_grad.push_back(dalloc<float>(P * 4));
            w->gp_ptrs = dalloc<const float *>(sizeof(float *) * w->k);
            CK(cudaMemcpy(w->gp_ptrs, w->gp_grad.data(), sizeof(float *) * w->k, cudaMemcpyHostToDevice));
            std::vector<float *> f32(w->k);
            std::vector<__nv_bfloat16 *> b16(w->k);
            for (int q = 0; q < w->k; ++q) {
                f32[q] = bf16 ? w->master : static_cast<float *>(w->wslot[q]);
                b16[q] = bf16 ? static_cast<__nv_bfloat16 *>(w->wslot[q]) : nullptr;
            }
            w->gp_out_f32 = dalloc<float *>(sizeof(float *) * w->k);
            w->gp_out_bf16 = dalloc<__nv_bfloat16 *>(sizeof(void *) * w->k);
            CK(cudaMemcpy(w->gp_out_f32, f32.data(), sizeof(float *) * w->k, cudaMemcpyHostToDevice));
            CK(cudaMemcpy(w->gp_out_bf16, b16.data(), sizeof(void *) * w->k, cudaMemcpyHostToDevice));
        }
        if (Rs > 1) {
            w->rgrad[0] = dalloc<float>(P * 4);
            w->rgrad[1] = dalloc<float>(P * 4);
            w->rgrad_ptrs = dalloc<const float *>(sizeof(float *) * 2 * Rs);
            if (w->k > MAX_SYNC_SLOTS) throw CudaFail{cudaErrorInvalidValue, "too many stash slots on a replicated stage"};
            w->sync_f32 = dalloc<float *>(sizeof(float *) * w->k * Rs);
            w->sync_bf16 = dalloc<__nv_bfloat16 *>(sizeof(void *) * w->k * Rs);
        }
        // activation stash for inner layers
        w->act.assign(w->last - w->first + 1, nullptr);
        long max_elems = 0;
        for (int l = w->first; l <= w->last; ++l) {
            max_elems = std::max(max_elems, std::max(dev_in_elems(c->layers, l, B), dev_out_elems(c->layers, l, B)));
            if (l > w->first) w->act[l - w->first] = dalloc<void>((size_t)w->k * dev_in_elems(c->layers, l, B) * esz);
        }
        w->scratch[0] = dalloc<void>(max_elems * esz);
        w->scratch[1] = dalloc<void>(max_elems * esz);
        w->scratch[2] = dalloc<void>(max_elems * esz);
        CK(cudaStreamCreateWithFlags(&w->side, cudaStreamNonBlocking));
        w->ev_dx.resize(w->last - w->first + 1);
        w->ev_dw.resize(w->last - w->first + 1);
        for (auto &e : w->ev_dx) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
        for (auto &e : w->ev_dw) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
        CK(cudaEventCreateWithFlags(&w->ev_fork, cudaEventDisableTiming));
        w->aux.assign(w->last - w->first + 1, nullptr);
        w->aux_bytes.assign(w->last - w->first + 1, 0);
        long gx_elems = 0, bh_elems = 0;
        for (int l = w->first; l <= w->last; ++l) {
            const pd_layer_desc &d = c->layers[l];
            if (d.kind != PD_LSTM) continue;
            const long TB = (long)d.seq_len * B, H = d.out;
            const long bytes = align_up(TB * 4 * H * 4, 256) + align_up(TB * H * 4, 256) + align_up(TB * H * esz, 256);
            w->aux_bytes[l - w->first] = bytes;
            w->aux[l - w->first] = dalloc<void>((size_t)w->k * bytes);
            gx_elems = std::max(gx_elems, TB * 4 * H);
            bh_elems = std::max(bh_elems, (long)B * H);
        }
        // wavefront backward scratch (da and the dc carry of every layer of the longest chain of
        // equal LSTMs this stage can run as one wavefront), allocated here: an allocation inside
        // pd_run would device-synchronise while another worker captures a graph
        if (bf16) {
            int chain = 1, longest = 1;
            for (int l = w->first + 1; l <= w->last; ++l) {
                const pd_layer_desc &p = c->layers[l - 1], &q = c->layers[l];
                const bool link = p.kind == PD_LSTM && q.kind == PD_LSTM && p.in == p.out && q.in == p.out &&
                                  q.out == p.out && q.seq_len == p.seq_len;
                chain = link ? chain + 1 : 1;
                longest = std::max(longest, chain);
            }
            if (longest >= 2) {
                long tb4h = 0, bh = 0;  // the largest LSTM of the stage bounds every run's per-layer scratch
                for (int l = w->first; l <= w->last; ++l)
                    if (c->layers[l].kind == PD_LSTM) {
                        tb4h = std::max(tb4h, (long)c->layers[l].seq_len * B * 4 * c->layers[l].out);
                        bh = std::max(bh, (long)B * c->layers[l].out);
                    }
                w->lstm_wmax = std::min(longest, LSTM_WAVE_MAX_L);
                w->lstm_wda = dalloc<void>((size_t)w->lstm_wmax * tb4h * esz);
                w->lstm_wdc = dalloc<float>((size_t)w->lstm_wmax * bh * 4);
                for (int i = 0; i < 6; ++i) {
                    CK(cudaStreamCreateWithFlags(&w->dw_stream[i], cudaStreamNonBlocking));
                    CK(cudaEventCreateWithFlags(&w->dw_ev[i], cudaEventDisableTiming));
                }
                CK(cudaHostAlloc(reinterpret_cast<void **>(&w->wave_flag), 64, cudaHostAllocMapped));
                *w->wave_flag = 0;
            }
        }
        if (gx_elems) {
            w->lstm_gx = dalloc<float>(gx_elems * 4);
            w->lstm_da = dalloc<void>(gx_elems * esz);
            w->lstm_gh = dalloc<float>(4 * bh_elems * 4);
            w->lstm_dh = dalloc<float>(bh_elems * 4);
            w->lstm_dc = dalloc<float>(bh_elems * 4);
            w->lstm_cnt = dalloc<unsigned>(1024 * sizeof(unsigned));
        }
        if (bf16) {
            w->ws_bytes = 8L * max_elems * 4;  // up to 8 K-splits of the widest activation
            w->ws = dalloc<float>(w->ws_bytes);
            w->loss_scratch = dalloc<float>(256);
        }
        if (stage > 0) w->recv = dalloc<void>((size_t)w->D * dev_in_elems(c->layers, w->first, B) * esz);
        if (stage + 1 < c->n) w->gring = dalloc<void>((size_t)w->G * dev_out_elems(c->layers, w->last, B) * esz);
        if (stage + 1 == c->n) {
            const long lo = out_elems(c->layers[w->last], B);
            w->logits = dalloc<void>(lo * esz);
            w->dlogits = dalloc<void>(lo * esz);
        }
        w->flags = dalloc<uint32_t>(sizeof(uint32_t) * std::max(1, c->flag_count(stage)));
        CK(cudaDeviceSynchronize());
        // the worker's shareable buffers
        Shared &sh = c->shared[id];
        sh.recv = w->recv;
        sh.grad = w->gring;
        sh.rgrad[0] = w->rgrad[0];
        sh.rgrad[1] = w->rgrad[1];
        if (Rs > 1) {
            sh.nslots = w->k;
            for (int q = 0; q < w->k; ++q) sh.wslot[q] = w->wslot[q];
            sh.master = w->master;
        }
        sh.flags = w->flags;
        sh.valid = true;
    } catch (const CudaFail &f) {
        cudaGetLastError();
        c->shared[id] = Shared{};
        return f.e == cudaErrorMemoryAllocation ? PD_ENOMEM : PD_ECUDA;
    }
    c->W[id] = std::move(w);
    return PD_OK;
}

pd_status pd_export_worker(pd_ctx *c, int stage, int replica, void *blob, size_t cap, size_t *len) {
    CHECK_CTX(c);
    if (!len || stage < 0 || stage >= c->n || replica < 0 || replica >= c->plan.stage[stage].replicas) return PD_EINVAL;
    *len = sizeof(IpcBlob);
    const int id = c->worker_id(stage, replica);
    Worker *w = c->W[id].get();
    if (!w || !blob || cap < sizeof(IpcBlob)) return PD_EINVAL;
    IpcBlob b{};
    b.magic = BLOB_MAGIC;
    b.stage = stage;
    b.replica = replica;
    b.device = w->device;
    if (cudaSetDevice(w->device) != cudaSuccess) return PD_ECUDA;
    if (w->recv) {
        b.has_recv = 1;
        if (cudaIpcGetMemHandle(&b.recv, w->recv) != cudaSuccess) return PD_ECUDA;
    }
    if (w->gring) {
        b.has_grad = 1;
        if (cudaIpcGetMemHandle(&b.grad, w->gring) != cudaSuccess) return PD_ECUDA;
    }
    if (w->rgrad[0]) {
        b.has_rgrad = 1;
        if (cudaIpcGetMemHandle(&b.rgrad0, w->rgrad[0]) != cudaSuccess) return PD_ECUDA;
        if (cudaIpcGetMemHandle(&b.rgrad1, w->rgrad[1]) != cudaSuccess) return PD_ECUDA;
        b.nslots = w->k;
        for (int q = 0; q < w->k; ++q)
            if (cudaIpcGetMemHandle(&b.wslot[q], w->wslot[q]) != cudaSuccess) return PD_ECUDA;
        if (w->master) {
            b.has_master = 1;
            if (cudaIpcGetMemHandle(&b.master, w->master) != cudaSuccess) return PD_ECUDA;
        }
    }
    if (cudaIpcGetMemHandle(&b.flags, w->flags) != cudaSuccess) return PD_ECUDA;
    std::memcpy(blob, &b, sizeof b);
    return PD_OK;
}

pd_status pd_import_worker(pd_ctx *c, const void *blob, size_t len) {
    CHECK_CTX(c);
    if (!blob || len < sizeof(IpcBlob)) return PD_EINVAL;
    IpcBlob b;
    std::memcpy(&b, blob, sizeof b);
    if (b.magic != BLOB_MAGIC || b.stage < 0 || b.stage >= c->n || b.replica < 0 ||
        b.replica >= c->plan.stage[b.stage].replicas)
        return PD_EINVAL;
    const int id = c->worker_id(b.stage, b.replica);
    if (c->W[id]) return PD_EINVAL;  // local worker
    if (c->shared[id].valid) return PD_OK;
    // map into the device of a local worker (any; peer pointers are UVA)
    int dev = -1;
    for (auto &w : c->W)
        if (w) { dev = w->device; break; }
    if (dev < 0) return PD_ESTATE;
    if (cudaSetDevice(dev) != cudaSuccess) return PD_ECUDA;
    Shared sh;
    auto open = [&](const cudaIpcMemHandle_t &h, void **p) {
        return cudaIpcOpenMemHandle(p, h, cudaIpcMemLazyEnablePeerAccess) == cudaSuccess;
    };
    bool ok = true;
    if (b.has_recv) ok = ok && open(b.recv, &sh.recv);
    if (b.has_grad) ok = ok && open(b.grad, &sh.grad);
    if (b.has_rgrad) {
        ok = ok && open(b.rgrad0, reinterpret_cast<void **>(&sh.rgrad[0]));
        ok = ok && open(b.rgrad1, reinterpret_cast<void **>(&sh.rgrad[1]));
        if (b.nslots < 0 || b.nslots > MAX_SYNC_SLOTS) ok = false;
        sh.nslots = ok ? b.nslots : 0;
        for (int q = 0; q < sh.nslots; ++q) ok = ok && open(b.wslot[q], &sh.wslot[q]);
        if (b.has_master) ok = ok && open(b.master, reinterpret_cast<void **>(&sh.master));
    }
    ok = ok && open(b.flags, reinterpret_cast<void **>(&sh.flags));
    if (!ok) {
        cudaGetLastError();
        return PD_ECUDA;
    }
    sh.valid = true;
    c->shared[id] = sh;
    return PD_OK;
}

pd_status pd_set_data(pd_ctx *c, const float *inputs, const int32_t *tokens, const int32_t *labels, int nd) {
    CHECK_CTX(c);
    if (nd < 1) return PD_EINVAL;
    const int B = c->cfg.minibatch;
    const pd_layer_desc &L0 = c->layers.front();
    const pd_layer_desc &LL = c->layers.back();
    const bool emb = L0.kind == PD_EMBEDDING;
    if (emb ? !tokens : !inputs) return PD_EINVAL;
    if (!labels) return PD_EINVAL;
    const long in_n = in_elems(L0, B), rows = rows_of(LL, B);
    try {
        for (auto &wp : c->W) {
            Worker *w = wp.get();
            if (!w) continue;
            CK(cudaSetDevice(w->device));
            if (w->stage == 0) {
                if (emb) {
                    if (c->n_data != nd || !w->tokens) {
                        if (w->tokens) cudaFree(w->tokens);
                        w->tokens = dalloc<int32_t>((size_t)nd * in_n * 4);
                    }
                    CK(cudaMemcpyAsync(w->tokens, tokens, (size_t)nd * in_n * 4, cudaMemcpyHostToDevice, w->stream));
                } else {
                    const long dev_n = dev_in_elems(c->layers, 0, B);  // padded for a conv first layer
                    if (c->n_data != nd || !w->data_in) {
                        if (w->data_in) cudaFree(w->data_in);
                        w->data_in = dalloc<void>((size_t)nd * dev_n * c->esz);
                    }
                    if (c->esz == 4 && !padded_in(L0)) {
                        CK(cudaMemcpyAsync(w->data_in, inputs, (size_t)nd * in_n * 4, cudaMemcpyHostToDevice,
                                           w->stream));
                    } else {
                        // persistent fp32 staging (no allocation on the per-step path)
                        if (w->stage_in_elems < (long)nd * in_n) {
                            CK(cudaStreamSynchronize(w->stream));
                            if (w->stage_in) cudaFree(w->stage_in);
                            w->stage_in = dalloc<float>((size_t)nd * in_n * 4);
                            w->stage_in_elems = (long)nd * in_n;
                        }
                        CK(cudaMemcpyAsync(w->stage_in, inputs, (size_t)nd * in_n * 4, cudaMemcpyHostToDevice,
                                           w->stream));
                        if (padded_in(L0))
                            CK(pad_nhwc(w->stage_in, w->data_in, c->esz == 2, nd * B, L0.height, L0.width, L0.in,
                                        dev_channels(L0), w->stream));
                        else
                            CK(f32_to_bf16(w->stage_in, static_cast<__nv_bfloat16 *>(w->data_in), (long)nd * in_n,
                                           w->stream));
                    }
                }
            }
            if (w->stage + 1 == c->n) {
                if (c->n_data != nd || !w->labels) {
                    if (w->labels) cudaFree(w->labels);
                    w->labels = dalloc<int32_t>((size_t)nd * rows * 4);
                }
                CK(cudaMemcpyAsync(w->labels, labels, (size_t)nd * rows * 4, cudaMemcpyHostToDevice, w->stream));
            }
        }
    } catch (const CudaFail &f) {
        c->fail(PD_ECUDA, std::string("pd_set_data: ") + f.what + ": " + cudaGetErrorString(f.e));
        return PD_ECUDA;
    }
    c->n_data = nd;
    return PD_OK;
}

pd_status pd_run(pd_ctx *c, int M, int noam) {
    CHECK_CTX(c);
    if (M < 1) return PD_EINVAL;
    for (int s = 0; s < c->n; ++s)
        if (M % c->plan.stage[s].replicas) return PD_EINVAL;
    std::vector<int> k;
    const bool gpipe = c->cfg.sync_mode == PD_SYNC_GPIPE;
    if (gpipe) {
        // flush groups of D = noam (0 => NOAM = n) minibatches: k_s = D at every stage (a whole
        // group in flight; the last stage runs F B back to back), R27; Exec reads D as k[0]
        const int D = noam > 0 ? noam : c->n;
        if (M % D) return PD_EINVAL;
        k.assign(c->n, D);
        for (int s = 0; s < c->n; ++s)
            if (D > c->kalloc[s]) return PD_EINVAL;
    } else {
        if (inflight_counts(c->plan, noam, k) != PD_OK) return PD_EINVAL;
    }
    for (int s = 0; s < c->n; ++s)
        if (k[s] > c->kalloc[s]) return PD_EINVAL;
    if (c->n_data < 1) return PD_ESTATE;
    for (int id = 0; id < c->nw; ++id)
        if (!c->shared[id].valid) return PD_ESTATE;
    bool any_local = false;
    for (auto &w : c->W) any_local = any_local || (bool)w;
    if (!any_local) return PD_ESTATE;
    // with a depth override the stash ring must still hold k_s versions at every worker
    try {
        // links (created once; local when both ends are in this process)
        auto make_link = [&](int type, int src, int dst) {
            auto key = std::make_tuple(type, src, dst);
            if (c->links.count(key)) return;
            auto L = std::make_unique<Link>();
            Worker *ws = c->W[src].get(), *wd = c->W[dst].get();
            if (ws && wd) {
                L->remote = false;
                L->device = ws->device;
                CK(cudaSetDevice(ws->device));
                const int E = 2 * std::max(8, std::max(c->Dalloc[wd->stage], c->kalloc[ws->stage])) + 4;
                L->ev.resize(E);
                L->snap.resize(E);
                for (auto &e : L->ev) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
                if (ws->device != wd->device) {
                    int can = 0;
                    CK(cudaDeviceCanAccessPeer(&can, ws->device, wd->device));
                    if (can) {
                        cudaError_t e = cudaDeviceEnablePeerAccess(wd->device, 0);
                        if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) CK(e);
                        cudaGetLastError();
                        CK(cudaSetDevice(wd->device));
                        e = cudaDeviceEnablePeerAccess(ws->device, 0);
                        if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) CK(e);
                        cudaGetLastError();
                    }
                }
            } else {
                L->remote = true;
                const int ds = c->stage_of(dst), sst = c->stage_of(src);
                const int sr = src - c->wbase[sst];
                const int fi = c->flag_index(type, sst, sr, ds);
                if (ws) L->remote_flag = c->shared[dst].flags + fi;  // IPC-mapped
                if (wd) L->local_flag = wd->flags + fi;
            }
            c->links[key] = std::move(L);
        };
        for (int s = 0; s < c->n; ++s) {
            const int Rs = c->plan.stage[s].replicas;
            for (int r = 0; r < Rs; ++r) {
                const int id = c->worker_id(s, r);
                if (s + 1 < c->n) {
                    const int Rn = c->plan.stage[s + 1].replicas;
                    for (int q = 0; q < Rn; ++q) {
                        const int od = c->worker_id(s + 1, q);
                        if (c->W[id] || c->W[od]) {
                            make_link(L_ACT, id, od);
                            make_link(L_GRAD, od, id);
                        }
                    }
                }
                for (int q = 0; q < Rs; ++q) {
                    const int od = c->worker_id(s, q);
                    if (q != r && (c->W[id] || c->W[od])) {
                        make_link(L_READY, id, od);
                        make_link(L_DONE, id, od);
                    }
                }
            }
        }
        // reset the host-side counters of local links; remote flags are monotonic across
        // runs (no reset, so no cross-process barrier is needed before a run): the consumer's
        // base advances by what the producer posted in the previous run, which the static
        // schedule fixes -- activations / gradients: the minibatches routed from the source
        // replica to the destination replica; READY / DONE: one per round (M / R_s)
        for (auto &kv : c->links) {
            Link &L = *kv.second;
            L.posted = L.waited = 0;
            const int type = std::get<0>(kv.first), src = std::get<1>(kv.first), dst = std::get<2>(kv.first);
            const int ss = c->stage_of(src), ds = c->stage_of(dst);
            const int sr = src - c->wbase[ss], dr = dst - c->wbase[ds];
            int64_t msgs = 0;
            if (type == L_READY || type == L_DONE) {
                msgs = M / c->plan.stage[ss].replicas;
            } else {
                const int Rs = c->plan.stage[ss].replicas, Rd = c->plan.stage[ds].replicas;
                for (int t = 0; t < M; ++t) msgs += (t % Rs == sr && t % Rd == dr);
            }
            L.rbase += L.rcount;
            L.rcount = msgs;
        }
        // op indices of every worker's static list (slot-ownership checker)
        c->opF.assign(c->nw, {});
        c->opB.assign(c->nw, {});
        c->opU.assign(c->nw, {});
        for (int s = 0; s < c->n; ++s) {
            const int Rs = c->plan.stage[s].replicas;
            for (int r = 0; r < Rs; ++r) {
                const int id = c->worker_id(s, r);
                const std::vector<Op> ops = gpipe ? gpipe_ops(s + 1 == c->n, k[0], M) : worker_ops(Rs, r, k[s], M);
                const int Mr = M / Rs;
                c->opF[id].assign(Mr, -1);
                c->opB[id].assign(Mr, -1);
                c->opU[id].assign(Mr, -1);  // (GPipe: M / D updates, indexed by group)
                for (size_t i = 0; i < ops.size(); ++i)
                    (ops[i].kind == 'F' ? c->opF : ops[i].kind == 'B' ? c->opB : c->opU)[id][ops[i].j] = (int32_t)i;
            }
        }
        for (auto &wp : c->W) {
            Worker *w = wp.get();
            if (!w) continue;
            CK(cudaSetDevice(w->device));
            if (w->stage + 1 == c->n && w->losses_cap < M) {
                if (w->losses) cudaFree(w->losses);
                w->losses = dalloc<float>((size_t)M * 4);
                w->losses_cap = M;
            }
            if (w->stage + 1 == c->n) CK(cudaMemsetAsync(w->losses, 0, (size_t)M * 4, w->stream));
            const int Rs = c->plan.stage[w->stage].replicas;
            if (Rs > 1) {
                std::vector<const float *> ptrs(2 * Rs);
                for (int par = 0; par < 2; ++par)
                    for (int r = 0; r < Rs; ++r) ptrs[par * Rs + r] = c->shared[c->worker_id(w->stage, r)].rgrad[par];
                CK(cudaMemcpy(w->rgrad_ptrs, ptrs.data(), sizeof(float *) * ptrs.size(), cudaMemcpyHostToDevice));
                std::vector<float *> f32((size_t)w->k * Rs);
                std::vector<__nv_bfloat16 *> b16((size_t)w->k * Rs);
                for (int q = 0; q < w->k; ++q)
                    for (int r = 0; r < Rs; ++r) {
                        const Shared &ps = c->shared[c->worker_id(w->stage, r)];
                        if (ps.nslots != w->k) throw CudaFail{cudaErrorInvalidValue, "replica stash depth mismatch"};
                        if (c->esz == 2) {
                            f32[(size_t)q * Rs + r] = ps.master;
                            b16[(size_t)q * Rs + r] = static_cast<__nv_bfloat16 *>(ps.wslot[q]);
                        } else {
                            f32[(size_t)q * Rs + r] = static_cast<float *>(ps.wslot[q]);
                            b16[(size_t)q * Rs + r] = nullptr;
                        }
                    }
                CK(cudaMemcpy(w->sync_f32, f32.data(), sizeof(float *) * f32.size(), cudaMemcpyHostToDevice));
                CK(cudaMemcpy(w->sync_bf16, b16.data(), sizeof(void *) * b16.size(), cudaMemcpyHostToDevice));
            }
            w->events.clear();
            w->op_ev.clear();
            w->bytes_sent = w->replica_bytes = 0;
            for (auto &kv : w->kev) kv.clear();
            for (auto &e : w->run_ev)
                if (!e) CK(cudaEventCreate(&e));
            const int nl = w->last - w->first + 1;
            w->lev.clear();
            const size_t need = (c->cfg.record_trace >= 2 ? (size_t)(6 + 8 * nl) * M + 16 : 0) +
                                (c->layer_prof ? (size_t)4 * nl * M + 16 : 0);
            while (w->ev_pool.size() < need) {
                cudaEvent_t e;
                CK(cudaEventCreate(&e));
                w->ev_pool.push_back(e);
            }
            CK(cudaStreamSynchronize(w->stream));
            CK(cudaDeviceSynchronize());  // legacy-stream copies (rgrad_ptrs) before the run
        }
    } catch (const CudaFail &f) {
        c->fail(PD_ECUDA, std::string("pd_run setup: ") + f.what + ": " + cudaGetErrorString(f.e));
        return PD_ECUDA;
    }
    c->last_M = M;
    c->vmap.assign((size_t)c->n * M, -1);
    auto t0 = std::chrono::steady_clock::now();
    std::vector<std::thread> th;
    c->running = 0;
    for (auto &wp : c->W) c->running += wp ? 1 : 0;
    for (auto &wp : c->W)
        if (wp) {
            wp->st_where = 0;
            wp->st_op = -1;
            th.emplace_back(worker_thread, c, wp.get(), M, k);
        }
    // watchdog: a run that makes no progress for 60 s is reported once on stderr (per worker:
    // the op it issues and where its host thread waits) -- diagnosis only, it does not abort
    {
        const auto start = std::chrono::steady_clock::now();
        std::vector<int> last_op(c->nw, -2);
        auto last_change = start;
        bool reported = false;
        for (;;) {
            {
                std::unique_lock<std::mutex> g(c->done_mu);
                if (c->done_cv.wait_for(g, std::chrono::seconds(1), [&] { return c->running == 0; })) break;
            }
            bool changed = false;
            for (auto &wp : c->W)
                if (wp) {
                    const int op = wp->st_op.load();
                    if (op != last_op[wp->id]) last_op[wp->id] = op, changed = true;
                }
            const auto now = std::chrono::steady_clock::now();
            if (changed) last_change = now;
            if (!reported && now - last_change > std::chrono::seconds(60)) {
                reported = true;
                static const char *where[] = {"issuing", "link_post (ring full)", "link_wait", "stream sync", "done"};
                for (auto &wp : c->W)
                    if (wp) {
                        const int wh = wp->st_where.load();
                        fprintf(stderr, "[pd] watchdog: no progress for 60 s: worker %d (stage %d) op %d, %s (message %ld)\n",
                                wp->id, wp->stage, wp->st_op.load(), where[wh < 0 || wh > 4 ? 0 : wh],
                                (long)wp->st_link.load());
                    }
            }
        }
    }
    for (auto &t : th) t.join();
    c->host_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    if (c->sticky != PD_OK) return c->sticky;
    return PD_OK;
}

pd_status pd_stage_solo(pd_ctx *c) {
    CHECK_CTX(c);
    Worker *w0 = nullptr;
    for (auto &w : c->W)
        if (w) {
            w0 = w.get();
            break;
        }
    if (!w0) return PD_ESTATE;
    for (int id = 0; id < c->nw; ++id)
        if (!c->W[id] && c->shared[id].valid && !c->shared[id].standin) return PD_ESTATE;  // real peer imported
    const int B = c->cfg.minibatch, esz = c->esz;
    try {
        CK(cudaSetDevice(w0->device));
        auto own = [&](size_t bytes) {
            void *p = dalloc<void>(bytes);
            c->solo_bufs.push_back(p);
            return p;
        };
        for (int id = 0; id < c->nw; ++id) {
            if (c->W[id] || c->shared[id].valid) continue;
            const int s = c->stage_of(id);
            const int first = c->plan.stage[s].first_layer, last = c->plan.stage[s].last_layer;
            Shared sh;
            if (s > 0) sh.recv = own((size_t)c->Dalloc[s] * dev_in_elems(c->layers, first, B) * esz);
            if (s + 1 < c->n) sh.grad = own((size_t)c->Galloc[s] * dev_out_elems(c->layers, last, B) * esz);
            if (c->plan.stage[s].replicas > 1) {
                const long P = c->poff[last] + (long)align_up(c->pcount[last], 64);
                sh.rgrad[0] = static_cast<float *>(own((size_t)P * 4));
                sh.rgrad[1] = static_cast<float *>(own((size_t)P * 4));
                sh.nslots = c->kalloc[s];
                for (int q = 0; q < sh.nslots; ++q) sh.wslot[q] = own((size_t)P * esz);
                if (esz == 2) sh.master = static_cast<float *>(own((size_t)P * 4));
            }
            sh.flags = static_cast<uint32_t *>(own(sizeof(uint32_t) * std::max(1, c->flag_count(s))));
            sh.valid = sh.standin = true;
            c->shared[id] = sh;
        }
        // local workers: synthetic receive-ring contents, incoming flag words pre-posted
        for (auto &wp : c->W) {
            Worker *w = wp.get();
            if (!w) continue;
            CK(cudaSetDevice(w->device));
            if (w->recv)
                CK(fill_uniform(w->recv, (long)w->D * dev_in_elems(c->layers, w->first, B), esz == 2, 1.f,
                                0x5EED0000u + w->id, w->stream));
            if (w->gring)
                CK(fill_uniform(w->gring, (long)w->G * dev_out_elems(c->layers, w->last, B), esz == 2, 1e-3f,
                                0x5EED1000u + w->id, w->stream));
            CK(cudaMemsetAsync(w->flags, 0x7F, sizeof(uint32_t) * std::max(1, c->flag_count(w->stage)), w->stream));
            CK(cudaStreamSynchronize(w->stream));
        }
    } catch (const CudaFail &f) {
        c->fail(PD_ECUDA, std::string("pd_stage_solo: ") + f.what + ": " + cudaGetErrorString(f.e));
        return f.e == cudaErrorMemoryAllocation ? PD_ENOMEM : PD_ECUDA;
    }
    return PD_OK;
}

namespace {
struct CkptHeader {
    char magic[8];  // "PDCKPT1"
    int32_t stage, replica, dtype, optimizer;
    int32_t version, updates_total;
    int64_t params;  // device-layout parameter count of the stage (P)
    int32_t has_adam, pad;
};
std::string ckpt_path(const char *dir, int s, int r) {
    return std::string(dir) + "/stage" + std::to_string(s) + "_replica" + std::to_string(r) + ".pdckpt";
}
}  // namespace

pd_status pd_save_checkpoint(pd_ctx *c, const char *dir) {
    CHECK_CTX(c);
    if (!dir) return PD_EINVAL;
    for (auto &wp : c->W) {
        Worker *w = wp.get();
        if (!w) continue;
        const std::string path = ckpt_path(dir, w->stage, w->replica);
        if (cudaSetDevice(w->device) != cudaSuccess || cudaStreamSynchronize(w->stream) != cudaSuccess) {
            c->fail(PD_ECUDA, "pd_save_checkpoint: device");
            return PD_ECUDA;
        }
        const bool adam = c->cfg.optimizer == PD_ADAM;
        std::vector<float> buf((size_t)w->P * (adam ? 3 : 1));
        // the latest weights: the fp32 master (bf16 path) or the latest fp32 version slot
        const float *src = c->esz == 2 ? w->master : static_cast<const float *>(w->wslot[w->version % w->k]);
        bool ok = cudaMemcpyAsync(buf.data(), src, (size_t)w->P * 4, cudaMemcpyDeviceToHost, w->stream) == cudaSuccess;
        if (adam)
            ok = ok &&
                 cudaMemcpyAsync(buf.data() + w->P, w->adam_m, (size_t)w->P * 4, cudaMemcpyDeviceToHost, w->stream) ==
                     cudaSuccess &&
                 cudaMemcpyAsync(buf.data() + 2 * w->P, w->adam_v, (size_t)w->P * 4, cudaMemcpyDeviceToHost,
                                 w->stream) == cudaSuccess;
        ok = ok && cudaStreamSynchronize(w->stream) == cudaSuccess;
        if (!ok) {
            c->fail(PD_ECUDA, "pd_save_checkpoint: copy");
            return PD_ECUDA;
        }
        CkptHeader h{};
        std::memcpy(h.magic, "PDCKPT1", 8);
        h.stage = w->stage, h.replica = w->replica, h.dtype = c->cfg.dtype, h.optimizer = c->cfg.optimizer;
        h.version = w->version, h.updates_total = w->updates_total, h.params = w->P, h.has_adam = adam;
        FILE *f = fopen((path + ".tmp").c_str(), "wb");
        const bool wrote = f && fwrite(&h, sizeof h, 1, f) == 1 && fwrite(buf.data(), 4, buf.size(), f) == buf.size();
        if (f) fclose(f);
        if (!wrote || rename((path + ".tmp").c_str(), path.c_str()) != 0) {
            std::lock_guard<std::mutex> g(c->err_mu);
            c->err = "pd_save_checkpoint: cannot write " + path;
            return PD_EINVAL;
        }
    }
    return PD_OK;
}

pd_status pd_load_checkpoint(pd_ctx *c, const char *dir) {
    CHECK_CTX(c);
    if (!dir) return PD_EINVAL;
    for (auto &wp : c->W) {
        Worker *w = wp.get();
        if (!w) continue;
        const std::string path = ckpt_path(dir, w->stage, w->replica);
        const bool adam = c->cfg.optimizer == PD_ADAM;
        CkptHeader h{};
        std::vector<float> buf((size_t)w->P * (adam ? 3 : 1));
        FILE *f = fopen(path.c_str(), "rb");
        const bool read = f && fread(&h, sizeof h, 1, f) == 1 && std::memcmp(h.magic, "PDCKPT1", 8) == 0 &&
                          h.stage == w->stage && h.replica == w->replica && h.dtype == c->cfg.dtype &&
                          h.optimizer == c->cfg.optimizer && h.params == w->P && h.has_adam == (int)adam &&
                          fread(buf.data(), 4, buf.size(), f) == buf.size();
        if (f) fclose(f);
        if (!read) {
            std::lock_guard<std::mutex> g(c->err_mu);
            c->err = "pd_load_checkpoint: missing or mismatching " + path;
            return PD_EINVAL;
        }
        try {
            // every copy and conversion on the worker's stream: a pageable cudaMemcpy may return
            // before its DMA lands, and the conversion kernel must not read the master before
            CK(cudaSetDevice(w->device));
            CK(cudaStreamSynchronize(w->stream));
            if (c->esz == 2) {
                CK(cudaMemcpyAsync(w->master, buf.data(), (size_t)w->P * 4, cudaMemcpyHostToDevice, w->stream));
                for (void *slot : w->wslot)
                    CK(f32_to_bf16(w->master, static_cast<__nv_bfloat16 *>(slot), w->P, w->stream));
            } else {
                for (void *slot : w->wslot)
                    CK(cudaMemcpyAsync(slot, buf.data(), (size_t)w->P * 4, cudaMemcpyHostToDevice, w->stream));
            }
            if (adam) {
                CK(cudaMemcpyAsync(w->adam_m, buf.data() + w->P, (size_t)w->P * 4, cudaMemcpyHostToDevice, w->stream));
                CK(cudaMemcpyAsync(w->adam_v, buf.data() + 2 * w->P, (size_t)w->P * 4, cudaMemcpyHostToDevice,
                                   w->stream));
            }
            CK(cudaStreamSynchronize(w->stream));
        } catch (const CudaFail &e) {
            c->fail(PD_ECUDA, std::string("pd_load_checkpoint: ") + e.what);
            return PD_ECUDA;
        }
        w->version = h.version;
        w->updates_total = h.updates_total;
    }
    return PD_OK;
}

pd_status pd_get_params(pd_ctx *c, int layer, float *host_out, size_t count) {
    CHECK_CTX(c);
    if (layer < 0 || layer >= (int)c->layers.size() || !host_out) return PD_EINVAL;
    if (count != (size_t)c->hcount[layer]) return PD_EINVAL;
    int s = 0;
    while (c->plan.stage[s].last_layer < layer) ++s;
    Worker *w = nullptr;
    for (int r = 0; r < c->plan.stage[s].replicas && !w; ++r) w = c->W[c->worker_id(s, r)].get();
    if (!w) return PD_EINVAL;
    if (count == 0) return PD_OK;
    if (cudaSetDevice(w->device) != cudaSuccess) return PD_ECUDA;
    const float *src = (c->cfg.dtype == PD_BF16) ? w->master : static_cast<const float *>(w->wslot[w->version % w->k]);
    std::vector<float> dev(c->pcount[layer]);
    if (cudaMemcpy(dev.data(), src + c->poff[layer], dev.size() * 4, cudaMemcpyDeviceToHost) != cudaSuccess) {
        c->fail(PD_ECUDA, "pd_get_params copy");
        return PD_ECUDA;
    }
    params_from_dev(c->layers[layer], dev.data(), host_out);
    return PD_OK;
}

pd_status pd_get_trace(pd_ctx *c, pd_event *out, size_t cap, size_t *written) {
    CHECK_CTX(c);
    if (!written) return PD_EINVAL;
    size_t total = 0;
    for (auto &w : c->W)
        if (w) total += w->events.size();
    *written = total;
    if (!out) return PD_OK;
    if (cap < total) return PD_EINVAL;
    size_t i = 0;
    for (auto &wp : c->W) {
        Worker *w = wp.get();
        if (!w) continue;
        const bool timed = c->cfg.record_trace >= 2 && w->op_ev.size() * 3 >= w->events.size() * 2;
        size_t opi = 0;
        for (auto &e : w->events) {
            pd_event x = e;
            if (timed && e.kind != 'U' && opi < w->op_ev.size() && w->op_ev[opi].second) {
                float a = 0, b = 0;
                cudaSetDevice(w->device);
                if (cudaEventElapsedTime(&a, w->op_ev[0].first, w->op_ev[opi].first) == cudaSuccess &&
                    cudaEventElapsedTime(&b, w->op_ev[0].first, w->op_ev[opi].second) == cudaSuccess) {
                    x.start_us = a * 1000.f;
                    x.end_us = b * 1000.f;
                }
                ++opi;
            }
            out[i++] = x;
        }
    }
    return PD_OK;
}

pd_status pd_get_version_map(pd_ctx *c, int32_t *out, size_t cap) {
    CHECK_CTX(c);
    if (!out || cap < c->vmap.size()) return PD_EINVAL;
    std::memcpy(out, c->vmap.data(), c->vmap.size() * 4);
    return PD_OK;
}

pd_status pd_get_losses(pd_ctx *c, float *out, size_t cap) {
    CHECK_CTX(c);
    if (!out || cap < (size_t)c->last_M) return PD_EINVAL;
    for (int t = 0; t < c->last_M; ++t) out[t] = NAN;
    for (auto &wp : c->W) {
        Worker *w = wp.get();
        if (!w || w->stage + 1 != c->n || !w->losses) continue;
        std::vector<float> tmp(c->last_M);
        if (cudaSetDevice(w->device) != cudaSuccess ||
            cudaMemcpy(tmp.data(), w->losses, (size_t)c->last_M * 4, cudaMemcpyDeviceToHost) != cudaSuccess) {
            c->fail(PD_ECUDA, "pd_get_losses copy");
            return PD_ECUDA;
        }
        const int Rs = c->plan.stage[w->stage].replicas;
        for (int t = w->replica; t < c->last_M; t += Rs) out[t] = tmp[t];
    }
    return PD_OK;
}

pd_status pd_get_stats(pd_ctx *c, pd_stats *out) {
    CHECK_CTX(c);
    if (!out) return PD_EINVAL;
    std::memset(out, 0, sizeof *out);
    out->host_ms = c->host_ms;
    double busy_sum = 0, span_max = 0;
    int nl = 0;
    for (auto &wp : c->W) {
        Worker *w = wp.get();
        if (!w) continue;
        out->kernel_launches += w->launches;
        out->bytes_sent += w->bytes_sent;
        out->replica_bytes += w->replica_bytes;
        double busy = 0, span = 0;
        if (!w->op_ev.empty() && w->op_ev.back().second) {
            cudaSetDevice(w->device);
            for (auto &pr : w->op_ev) {
                float ms = 0;
                if (pr.second && cudaEventElapsedTime(&ms, pr.first, pr.second) == cudaSuccess) busy += ms;
            }
            float sp = 0;
            if (cudaEventElapsedTime(&sp, w->op_ev.front().first, w->op_ev.back().second) == cudaSuccess) span = sp;
        }
        float run_ms = 0;
        if (w->run_ev[0] && cudaEventElapsedTime(&run_ms, w->run_ev[0], w->run_ev[1]) == cudaSuccess)
            out->run_ms = std::max(out->run_ms, (double)run_ms);
        cudaGetLastError();
        for (int cls = 0; cls < PD_KERNEL_CLASSES; ++cls)
            for (auto &pr : w->kev[cls]) {
                float ms = 0;
                if (cudaEventElapsedTime(&ms, pr.first, pr.second) == cudaSuccess) {
                    out->kern_ms[cls] += ms;
                    out->kern_count[cls] += 1;
                }
            }
        if (nl < PD_MAX_LOCAL_WORKERS) {
            out->worker_id[nl] = w->id;
            out->busy_ms[nl] = busy;
            out->span_ms[nl] = span;
        }
        busy_sum += busy;
        span_max = std::max(span_max, span);
        ++nl;
    }
    out->num_local_workers = nl;
    out->device_ms = span_max;
    out->bubble = (span_max > 0 && nl > 0) ? 1.0 - busy_sum / (nl * span_max) : 0.0;
    return PD_OK;
}

pd_status pd_set_timing(pd_ctx *c, int record_trace, int mask) {
    CHECK_CTX(c);
    if (record_trace < 0 || record_trace > 2) return PD_EINVAL;
    c->cfg.record_trace = record_trace;
    c->ktime_mask = mask & ((1 << PD_KERNEL_CLASSES) - 1);
    return PD_OK;
}

pd_status pd_set_layer_profiling(pd_ctx *c, int on) {
    CHECK_CTX(c);
    c->layer_prof = on ? 1 : 0;
    return PD_OK;
}

pd_status pd_get_layer_times(pd_ctx *c, double *fwd_s, double *bwd_s, size_t count) {
    CHECK_CTX(c);
    if (!fwd_s || !bwd_s || count != c->layers.size()) return PD_EINVAL;
    std::vector<double> f(count, 0.0), b(count, 0.0);
    std::vector<int> nf(count, 0), nb(count, 0);
    for (auto &wp : c->W) {
        Worker *w = wp.get();
        if (!w) continue;
        if (cudaSetDevice(w->device) != cudaSuccess) return PD_ECUDA;
        for (auto &e : w->lev) {
            float ms = 0.f;
            if (cudaEventElapsedTime(&ms, e.a, e.b) != cudaSuccess) {
                c->fail(PD_ECUDA, "pd_get_layer_times: event elapsed time");
                return PD_ECUDA;
            }
            if (e.dir == 'F') f[e.layer] += ms * 1e-3, ++nf[e.layer];
            else b[e.layer] += ms * 1e-3, ++nb[e.layer];
        }
    }
    for (size_t l = 0; l < count; ++l) {
        fwd_s[l] = nf[l] ? f[l] / nf[l] : 0.0;
        bwd_s[l] = nb[l] ? b[l] / nb[l] : 0.0;
    }
    return PD_OK;
}

// The self-profiler: one single-stage (plain SGD/Adam, k = 1) pipeline of the whole model on
// `cuda_device`, synthetic inputs, per-layer events around every layer's forward (+ loss on
// the last layer) and backward (+ its fused weight update).
pd_status pd_profile(const pd_layer_desc *layers, int num_layers, const pd_train_cfg *cfg_in, int cuda_device,
                     int num_minibatches, pd_layer_profile *out) {
    if (!layers || num_layers < 1 || !cfg_in || !out || num_minibatches < 1 || cuda_device < 0) return PD_EINVAL;
    pd_plan_t plan{};
    plan.num_stages = 1;
    plan.stage[0] = {0, num_layers - 1, 1, 0};
    plan.noam = 1;
    pd_train_cfg cfg = *cfg_in;
    cfg.record_trace = 0;
    cfg.max_depth = 0;
    cfg.sync_mode = PD_SYNC_STASH;
    pd_ctx *c = nullptr;
    pd_status st = pd_create(&c, &plan, layers, num_layers, &cfg);
    if (st != PD_OK) return st;
    // deterministic small parameters / inputs (a counter hash; values only need to be finite)
    auto val = [](uint64_t i, float scale) {
        uint64_t x = i * 0x9E3779B97F4A7C15ull;
        x ^= x >> 29;
        return scale * ((float)(x % 2001) / 1000.f - 1.f);
    };
    std::vector<std::vector<float>> p(num_layers);
    std::vector<const float *> pp(num_layers, nullptr);
    for (int l = 0; l < num_layers; ++l) {
        const pd_layer_desc &d = layers[l];
        const int fan = d.kind == PD_LSTM ? d.out : d.kind == PD_CONV3X3 ? 9 * d.in : d.in;
        p[l].resize((size_t)c->hcount[l]);
        for (size_t i = 0; i < p[l].size(); ++i) p[l][i] = val(i + 7919ull * l, 1.f / std::sqrt((float)std::max(fan, 1)));
        pp[l] = p[l].empty() ? nullptr : p[l].data();
    }
    const int B = cfg.minibatch, nd = 2;
    const long in_n = in_elems(layers[0], B), rows = rows_of(layers[num_layers - 1], B);
    std::vector<float> x((size_t)nd * in_n);
    std::vector<int32_t> tok((size_t)nd * in_n), lab((size_t)nd * rows);
    for (size_t i = 0; i < x.size(); ++i) x[i] = val(i, 1.f);
    for (size_t i = 0; i < tok.size(); ++i) tok[i] = (int32_t)(i % (size_t)std::max(layers[0].in, 1));
    for (size_t i = 0; i < lab.size(); ++i) lab[i] = (int32_t)(i % (size_t)std::max(layers[num_layers - 1].out, 1));
    const bool emb = layers[0].kind == PD_EMBEDDING;
    std::vector<double> f(num_layers), b(num_layers);
    if ((st = pd_stage_init(c, 0, 0, cuda_device, pp.data())) == PD_OK &&
        (st = pd_set_data(c, emb ? nullptr : x.data(), emb ? tok.data() : nullptr, lab.data(), nd)) == PD_OK &&
        (st = pd_run(c, 2, 0)) == PD_OK &&  // warm-up: allocations, tensor maps, graphs
        (st = pd_set_layer_profiling(c, 1)) == PD_OK && (st = pd_run(c, num_minibatches, 0)) == PD_OK &&
        (st = pd_get_layer_times(c, f.data(), b.data(), num_layers)) == PD_OK) {
        const uint64_t esz = cfg.dtype == PD_BF16 ? 2 : 4;
        for (int l = 0; l < num_layers; ++l) {
            out[l].compute_s = f[l] + b[l];
            out[l].act_bytes = (uint64_t)out_elems(layers[l], B) * esz;
            out[l].param_bytes = (uint64_t)numel_params(layers[l]) * 4;  // fp32 gradients of the replica sync
        }
    }
    pd_destroy(c);
    return st;
}

void pd_destroy(pd_ctx *c) {
    if (!c) return;
    for (auto &w : c->W)
        if (w) {
            cudaSetDevice(w->device);
            cudaStreamSynchronize(w->stream);
        }
    for (auto &kv : c->links)
        for (auto e : kv.second->ev) cudaEventDestroy(e);
    c->links.clear();
    for (void *p : c->solo_bufs) cudaFree(p);
    for (int id = 0; id < c->nw; ++id) {
        if (c->W[id] || !c->shared[id].valid || c->shared[id].standin) continue;
        Shared &sh = c->shared[id];
        void *ps[] = {sh.recv, sh.grad, sh.rgrad[0], sh.rgrad[1], sh.flags, sh.master};
        for (void *p : ps)
            if (p) cudaIpcCloseMemHandle(p);
        for (int q = 0; q < sh.nslots; ++q)
            if (sh.wslot[q]) cudaIpcCloseMemHandle(sh.wslot[q]);
    }
    c->W.clear();
    delete c;
}

}  // extern "C"

// ================================================================== kernel-level C ABI
#include "../../include/pipedream_kernels.h"

extern "C" PD_API pd_status pd_kernel_gemm(const pd_gemm_desc *d, void *stream) {
    if (!d || d->M < 1 || d->N < 1 || d->K < 1 || !d->A || !d->B) return PD_EINVAL;
    if (d->epilogue < PD_EPI_STORE || d->epilogue > PD_EPI_ADAM) return PD_EINVAL;
    if (d->dtype == PD_FP32 && d->epilogue > PD_EPI_F32) return PD_EINVAL;
    Gemm g;
    g.M = d->M; g.N = d->N; g.K = d->K;
    g.A = d->A; g.lda = d->lda; g.amaj = d->a_mn_major ? MNMAJ : KMAJ;
    g.B = d->B; g.ldb = d->ldb; g.bmaj = d->b_mn_major ? MNMAJ : KMAJ;
    g.epi = d->epilogue;
    g.out = d->out; g.ldo = d->ldo;
    g.bias = d->bias; g.relu = d->relu;
    g.mask = d->mask; g.ldm = d->ldm;
    g.master = d->master; g.slot = d->slot; g.adam_m = d->adam_m; g.adam_v = d->adam_v;
    g.lr = d->lr; g.b1 = d->beta1; g.b2 = d->beta2; g.eps = d->eps; g.step = d->step;
    g.workspace = d->workspace; g.workspace_bytes = d->workspace_bytes;
    g.ws_zeroed = d->workspace_zeroed;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    cudaError_t e = d->dtype == PD_BF16 ? gemm_bf16(g, s) : gemm_f32(g, s);
    if (e == cudaErrorInvalidValue) return PD_EINVAL;
    return e == cudaSuccess ? PD_OK : PD_ECUDA;
}

extern "C" PD_API pd_status pd_kernel_bias_grad(int dtype, const void *G, long rows, long cols, float *grad_out,
                                                float *master, void *slot_bf16, int optimizer, float *m, float *v,
                                                float lr, float beta1, float beta2, float eps, int step, void *stream) {
    if (!G || rows < 1 || cols < 1 || (!grad_out && !master) || (master && dtype != PD_BF16) ||
        (master && optimizer == PD_ADAM && (!m || !v)))
        return PD_EINVAL;
    cudaError_t e = bias_grad(G, dtype == PD_BF16, rows, cols, grad_out, master, static_cast<__nv_bfloat16 *>(slot_bf16),
                              optimizer, m, v, lr, beta1, beta2, eps, step, static_cast<cudaStream_t>(stream));
    return e == cudaSuccess ? PD_OK : PD_ECUDA;
}

extern "C" PD_API pd_status pd_kernel_softmax_ce(int dtype, const void *logits, const int32_t *labels, long rows,
                                                 int C, void *dlogits, float *loss, void *stream) {
    if (!logits || !labels || !dlogits || !loss || rows < 1 || C < 1) return PD_EINVAL;
    cudaError_t e = softmax_ce(logits, dtype == PD_BF16, labels, rows, C, dlogits, loss,
                               static_cast<cudaStream_t>(stream));
    return e == cudaSuccess ? PD_OK : PD_ECUDA;
}

extern "C" PD_API pd_status pd_kernel_lstm_rec(const pd_lstm_rec_desc *d, void *stream) {
    if (!d || d->T < 1 || !d->w_hh || !d->counters || !d->gates || !d->c) return PD_EINVAL;
    if (d->direction != 0 && d->direction != 1) return PD_EINVAL;
    if (d->direction == 0 && (!d->gx || !d->b_ih || !d->b_hh || !d->h)) return PD_EINVAL;
    if (d->direction == 1 && (!d->dy || !d->da)) return PD_EINVAL;
    if (!lstm_rec_supported(d->B, d->H)) return PD_EUNSUPPORTED;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    if (cudaMemsetAsync(d->counters, 0, (size_t)(4 * d->H / 64) * sizeof(unsigned), s) != cudaSuccess)
        return PD_ECUDA;
    const __nv_bfloat16 *W = static_cast<const __nv_bfloat16 *>(d->w_hh);
    cudaError_t e =
        d->direction == 0
            ? lstm_rec_fwd(d->gx, d->b_ih, d->b_hh, W, d->gates, d->c, static_cast<__nv_bfloat16 *>(d->h),
                           d->counters, d->T, d->B, d->H, s, d->probe)
            : lstm_rec_bwd(static_cast<const __nv_bfloat16 *>(d->dy), d->gates, d->c, W,
                           static_cast<__nv_bfloat16 *>(d->da), d->counters, d->T, d->B, d->H, s, d->probe);
    return e == cudaSuccess ? PD_OK : PD_ECUDA;
}
