/*
 * pipedream.h -- C ABI of the B200-native PipeDream hot path (libpipedream.so).
 *
 * Method: Narayanan et al., "PipeDream: Generalized Pipeline Parallelism for DNN Training",
 * SOSP'19 (/root/reference/PAPER.md, cited as L<line>).  The library implements the
 * steady-state 1F1B-RR pipeline with weight stashing (§3.2-3.3), its runtime
 * state policies (§4) and the §3.1 partitioner (L841-985).  Readings of
 * silent / garbled passages are numbered R1..R24 in DESIGN.md.
 *
 * Conventions (all calls):
 *   - every function returns pd_status (0 == PD_OK) unless stated otherwise;
 *   - the CALLER owns every host pointer; the library copies in (pd_stage_init,
 *     pd_set_data) and copies out (pd_get_*) and never keeps a host pointer;
 *   - the LIBRARY owns all device memory, streams, events and host threads it creates and
 *     frees them in pd_destroy;
 *   - input validation failures return PD_EINVAL with no side effects;
 *   - the first CUDA failure is latched in the context: every later call on that context
 *     returns PD_ESTATE until pd_destroy (pd_last_error() gives the message);
 *   - a pd_ctx is not thread-safe: call it from one host thread.
 *   - there is no CPU fallback: without a usable sm_100 device every device call fails
 *     with PD_ECUDA / PD_EUNSUPPORTED.
 */
#ifndef PIPEDREAM_H
#define PIPEDREAM_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(__GNUC__)
#define PD_API __attribute__((visibility("default")))
#else
#define PD_API
#endif

typedef enum {
    PD_OK = 0,
    PD_EINVAL = -1,        /* invalid argument (nothing changed)                         */
    PD_ENOMEM = -2,        /* device or host allocation failed                           */
    PD_ECUDA = -3,         /* CUDA runtime/driver error (latched)                        */
    PD_ENCCL = -4,         /* reserved (collective transport error)                      */
    PD_ESTATE = -5,        /* sticky earlier error, or call made in the wrong order      */
    PD_EUNSUPPORTED = -6,  /* layer kind / dtype / plan shape not supported on this path */
    PD_EINFEASIBLE = -7    /* pd_plan: no partition satisfies the constraints            */
} pd_status;

/* ======================================================================================
 * 1. Planner -- PAPER.md §3.1 "Partitioning Algorithm" (L855-985), profile of L841-853.
 * ====================================================================================== */

/* One profiled layer (L841-843): T_l = total forward+backward compute time in seconds,
 * a_l = bytes of the layer's output activation (= bytes of its input gradient),
 * w_l = bytes of the layer's parameters. */
typedef struct {
    double compute_s;
    uint64_t act_bytes;
    uint64_t param_bytes;
} pd_layer_profile;

#define PD_MAX_LEVELS 4

typedef struct {
    double bandwidth_Bps; /* B_1 of the single topology level (R13); <= 0 => 900e9 (NVLink 5)   */
    int max_replicas;     /* 0 = unconstrained; 1 = straight pipeline; k = at most k per stage  */
    int comm_model;       /* 0 = literal L903-927 formula (default), 1 = per-link ring (R11)    */
    /* Hierarchical topology (Fig. 7), lowest level first: level k = 1..num_levels
     * is level_size[k-1] components of level k-1 joined by links of level_bw[k-1] bytes/s
     * (level 0 = one GPU).  num_levels 0 = one level (level_size = num_gpus, level_bw =
     * bandwidth_Bps); otherwise the product of level_size must equal num_gpus.  The DP runs
     * from the lowest level up (A^k built on A^{k-1}); max_replicas bounds the replication
     * chosen at every level.  The plan comes back flattened: a level-k stage replicated m'
     * times over level-(k-1) components runs its layers' level-(k-1) plan inside each
     * component, so each of those sub-stages is one stage replicated m' x (its own factor).
     * first_gpu stays consecutive (R18); routing t mod R_s keeps a minibatch inside one
     * component if replica rho is placed on component rho mod m' (multi-node placement is
     * the caller's). */
    int num_levels;
    int level_size[PD_MAX_LEVELS];
    double level_bw[PD_MAX_LEVELS];
} pd_plan_opts;

#define PD_MAX_STAGES 64

typedef struct {
    int first_layer, last_layer; /* inclusive layer range of the stage                 */
    int replicas;                /* R_s, the stage's replication factor                */
    int first_gpu;               /* replicas occupy GPUs first_gpu .. first_gpu+R_s-1 (R18) */
} pd_stage_desc;

typedef struct {
    int num_stages;
    pd_stage_desc stage[PD_MAX_STAGES];
    int noam;               /* NUM_OPT_ACTIVE_MINIBATCHES = ceil(GPUs / R_0)  (L1021, R1) */
    double slowest_stage_s; /* A(0 -> N-1, GPUs): predicted time of the slowest stage    */
} pd_plan_t;

/* Runs the dynamic program A(i->j, m) of L927-975 (single level, R10-R16) on the host.
 *   layers[num_layers] : the profile, layer order = model order
 *   num_gpus           : m, every GPU is used (R13)
 *   opts               : may be NULL (defaults)
 *   out                : written on success only
 * Errors: PD_EINVAL (num_layers < 1 or > 4096, num_gpus < 1 or > 4096, NULL layers/out),
 *         PD_EINFEASIBLE (e.g. max_replicas = 1 with fewer layers than GPUs). */
PD_API pd_status pd_plan(const pd_layer_profile *layers, int num_layers, int num_gpus, const pd_plan_opts *opts,
                  pd_plan_t *out);

/* ======================================================================================
 * 2. Model and training description.  Parameter layout (the parity contract):
 *    LINEAR   W[out][in], b[out]                      (y = act(x W^T + b))
 *    LSTM     W_ih[4H][in], W_hh[4H][H], b_ih[4H], b_hh[4H], gates (i, f, g, o)
 *    CONV3X3  W[Cout][Cin][3][3], b[Cout]  (stride 1, zero pad 1, NHWC activations)
 *    EMBEDDING E[V][H]
 *    MAXPOOL2 (no parameters; 2x2 stride 2)
 * Activations are row-major [rows][features]; sequence models are time-major
 * ([T][B][features], tokens/labels [T][B]); images are NHWC.  The model's last layer
 * produces logits; the loss is the mean softmax cross-entropy over rows (L1217, R8).
 * ====================================================================================== */
typedef enum { PD_LINEAR = 0, PD_LSTM = 1, PD_CONV3X3 = 2, PD_MAXPOOL2 = 3, PD_EMBEDDING = 4 } pd_layer_kind;
typedef enum { PD_ACT_NONE = 0, PD_ACT_RELU = 1 } pd_act;

typedef struct {
    int kind;          /* pd_layer_kind                                                   */
    int in, out;       /* features (linear/lstm), channels (conv/pool), vocab V / H (embedding) */
    int act;           /* pd_act (linear, conv)                                            */
    int seq_len;       /* T for sequence layers (lstm, embedding, per-token linear); else 0 */
    int height, width; /* input spatial size (conv, pool); else 0                          */
} pd_layer_desc;

typedef enum { PD_FP32 = 0, PD_BF16 = 1 } pd_dtype;
typedef enum { PD_SGD = 0, PD_ADAM = 1 } pd_optimizer;
/* Weight-version semantics across stages (§3.3):
 *   PD_SYNC_STASH     weight stashing: F(s,t) uses stage s's latest version, B(s,t) the
 *                     version its F used (the default; w_s^(t-n+s) in L1237-1241);
 *   PD_SYNC_VERTICAL  vertical sync: the input stage tags minibatch t with its latest
 *                     version v and EVERY stage runs F(s,t) and B(s,t) with its own stashed
 *                     version v (L1175-1186; update rule L1247-1253).  Straight plans only
 *                     (every R_s = 1, else PD_EUNSUPPORTED); every stage keeps k_0 versions.
 *   PD_SYNC_GPIPE     the paper's comparison schedule (§5.4) with gradient
 *                     aggregation (L1277-1279): minibatches in flush groups of D (the pd_run
 *                     `noam` argument; 0 => NOAM = n).  Every stage but the last forwards the
 *                     whole group and then runs its backwards in t order (the last stage runs
 *                     F(t) B(t) back to back); each backward writes its weight gradient into
 *                     its own fp32 buffer, and one update per group applies the mean of the D
 *                     gradients (summed in t order, times 1/D) -- a pipeline flush per group,
 *                     one weight version per group (v(s,t) = floor(t/D), R27).
 *                     Straight plans only (else PD_EUNSUPPORTED); D <= max(n, cfg.max_depth)
 *                     and num_minibatches % D == 0 (else PD_EINVAL).  Trace: one 'U' per
 *                     group with minibatch = the group index. */
typedef enum { PD_SYNC_STASH = 0, PD_SYNC_VERTICAL = 1, PD_SYNC_GPIPE = 2 } pd_sync_mode;

typedef struct {
    int dtype;        /* PD_FP32: fp32 SIMT parity path (no tensor cores, tf32 off);
                         PD_BF16: bf16 tcgen05 path, bf16 weight versions + fp32 master (R21) */
    int optimizer;    /* PD_SGD (no momentum/decay) or PD_ADAM (bias-corrected), R9         */
    float lr, beta1, beta2, eps;
    int minibatch;    /* B, samples per minibatch                                         */
    int record_trace; /* 0 = off, 1 = event trace + version map, 2 = also per-op device times */
    int max_depth;    /* largest pd_run depth override that will be requested (0 = NOAM)   */
    int sync_mode;    /* pd_sync_mode (0 = weight stashing)                                */
} pd_train_cfg;

typedef struct pd_ctx pd_ctx;

/* Self-profiler (L841-847 "Profiler"), B200-native: measures the planner's profile on THIS
 * GPU.  Runs the whole model as one stage (plain SGD/Adam) on `cuda_device` for 2 warm-up
 * and `num_minibatches` timed minibatches of synthetic inputs, with CUDA events around each
 * layer's share of every forward (the loss counts to the last layer) and backward (dX, dW
 * and the fused weight update), serialised on one stream.
 *   out[l].compute_s   = mean forward + backward device seconds of layer l per minibatch (T_l)
 *   out[l].act_bytes   = bytes of layer l's output activation in cfg->dtype (a_l)
 *   out[l].param_bytes = 4 * parameters of layer l: the fp32 gradient bytes a replicated
 *                        stage exchanges per round (w_l)
 * cfg: dtype, optimizer, lr/betas/eps and minibatch are used; the rest is ignored.
 * Errors: PD_EINVAL (bad arguments or layer shapes), PD_EUNSUPPORTED, PD_ENOMEM, PD_ECUDA. */
PD_API pd_status pd_profile(const pd_layer_desc *layers, int num_layers, const pd_train_cfg *cfg,
                            int cuda_device, int num_minibatches, pd_layer_profile *out);


/* Creates a context for the whole plan.  Nothing touches a device until pd_stage_init.
 * Validation (PD_EINVAL): stages contiguous and covering layers 0..num_layers-1, each
 * R_s >= 1, layer shapes consistent (out of layer l == in of layer l+1 etc.), minibatch
 * >= 1, max_depth only on straight plans, plan->noam either 0 or exactly ceil(W / R_0) (the
 * value pd_plan / pd_inflight derive; anything else is rejected, not ignored).
 * PD_EUNSUPPORTED: layer kind / dtype combination not implemented. */
PD_API pd_status pd_create(pd_ctx **ctx, const pd_plan_t *plan, const pd_layer_desc *layers, int num_layers,
                    const pd_train_cfg *cfg);

/* Binds worker (stage, replica) to CUDA device `cuda_device` in this process, allocates its
 * state (weight-stash ring of k_s versions, fp32 master and optimizer state, activation
 * rings, receive rings, stream) and copies the initial parameters in.
 *   init_params[j] : host fp32 array of layer (first_layer + j) of the stage, in the layout
 *                    above (NULL entries allowed for parameter-free layers); copied.
 * Every worker of the plan must be initialised in exactly one process before pd_run.
 * Errors: PD_EINVAL (bad indices, already initialised), PD_ENOMEM, PD_ECUDA. */
PD_API pd_status pd_stage_init(pd_ctx *ctx, int stage, int replica, int cuda_device, const float *const *init_params);

/* Multi-process operation (one process per GPU, e.g. torchrun): after every process has
 * initialised its local workers, each exports a blob per local worker (CUDA IPC handles of
 * its receive rings, flags and replica buffers) and imports the blobs of every other
 * worker.  Blobs are plain bytes; their transport (e.g. torch.distributed all_gather) is
 * the caller's.  In a single process that owns every worker these calls are not needed.
 *   pd_export_worker : writes at most `cap` bytes to `blob`, sets *len.  PD_EINVAL if the
 *                      worker is not local or cap is too small (*len gives the size needed).
 *   pd_import_worker : PD_EINVAL on a malformed blob or a blob of a local worker.
 * A blob starts with {uint32 magic, int32 stage, int32 replica} (little-endian), so a caller can
 * skip its own workers' blobs without importing them. */
PD_API pd_status pd_export_worker(pd_ctx *ctx, int stage, int replica, void *blob, size_t cap, size_t *len);
PD_API pd_status pd_import_worker(pd_ctx *ctx, const void *blob, size_t len);

/* Copies num_minibatches minibatches of training data to the devices of the local workers
 * that need them (stage 0: inputs or tokens; last stage: labels).  Minibatch t of a run uses
 * data index t mod num_minibatches.
 *   inputs : fp32 [n][B * input features]  (NULL when the first layer is an embedding)
 *   tokens : int32 [n][T * B]               (NULL unless the first layer is an embedding)
 *   labels : int32 [n][rows]                (rows = B, or T * B for sequence models)
 * May be called again between runs (same n replaces in place).  Asynchronous with respect to
 * the host only if the host buffers are pinned; ordered before the next pd_run. */
PD_API pd_status pd_set_data(pd_ctx *ctx, const float *inputs, const int32_t *tokens, const int32_t *labels,
                      int num_minibatches);

/* Trains on minibatches t = 0 .. num_minibatches-1 with 1F1B-RR and weight stashing:
 * startup admits k_s minibatches per worker, steady state alternates B/F, then drains
 * (L1011-1065); minibatch t goes to replica t mod R_s (L1067-1099).  Blocking: returns when
 * every local worker's device work has completed.  Weight versions and optimizer state
 * persist across calls (a second pd_run continues training; minibatch ids restart at 0).
 *   noam : 0 => the plan's in-flight counts k_s = ceil(W_{>=s} / R_s) (NOAM = k_0, R2);
 *          D > 0 => depth override for straight plans, k_s = max(1, D - s), k_{n-1} = 1 (R19),
 *          requires D <= cfg.max_depth.
 * Slot ownership (L1349-1353): every rewrite of a ring slot (activation / gradient receive
 * slot, replica gradient buffer, weight-stash slot) is checked on the host to follow the
 * completion of the op that last reads the slot's previous content, through the vector
 * clocks the awaited messages carry (workers of this process); a violation fails the run
 * with PD_ESTATE and a "slot ownership: ..." message in pd_last_error.
 * Errors: PD_EINVAL (num_minibatches < 1 or not a multiple of every R_s, bad noam),
 *         PD_ESTATE (workers not all initialised / imported, no data, slot ownership
 *         violated), PD_ECUDA. */
PD_API pd_status pd_run(pd_ctx *ctx, int num_minibatches, int noam);

/* Solo measurement mode (SURVEY.md §8(d) per-stage table; throughput is set by the slowest
 * stage, L775-777): measures the local workers of a multi-stage plan on their own, as if
 * every absent neighbour were infinitely fast.  Every worker NOT initialised in this process
 * is replaced by library-owned stand-in buffers (receive rings, gradient ring, replica
 * buffers, flag words) on the device of the first local worker; the local workers' own
 * receive rings are filled with synthetic values (activations U(-1, 1), gradients
 * U(-1e-3, 1e-3)) and their incoming flag words are pre-posted, so each runs its static op
 * list (same kernels, same k_s, same transfers into the stand-ins) without waiting.  The
 * parameters and losses it produces are not training results.  Call after pd_stage_init of
 * the local workers and instead of pd_import_worker; then pd_set_data / pd_run as usual.
 * Errors: PD_ESTATE (no local worker, or a real peer was already imported), PD_ENOMEM,
 *         PD_ECUDA. */
PD_API pd_status pd_stage_solo(pd_ctx *ctx);

/* Per-stage checkpointing (L1407-1413): every LOCAL worker writes its own state to
 * `<dir>/stage<s>_replica<r>.pdckpt` -- the latest weights in fp32 (the master on the bf16
 * path), the Adam m and v, its version and update count -- with no coordination across
 * workers ("each stage dumps its model parameters locally").  Call between pd_run calls: a
 * run ends drained, so the latest version is the only live one.  pd_load_checkpoint restores
 * a context created with the same plan, layers and config (after pd_stage_init, before the
 * next pd_run): every version slot gets the checkpointed weights, training continues as if
 * uninterrupted (same versions, same optimizer step).  A worker whose file is missing or
 * does not match (stage, replica, parameter count, dtype, optimizer) fails the call.
 * Errors: PD_EINVAL (NULL dir, mismatching file), PD_ESTATE, PD_ECUDA, PD_ENOMEM; an I/O
 * failure returns PD_EINVAL with the path in pd_last_error. */
PD_API pd_status pd_save_checkpoint(pd_ctx *ctx, const char *dir);
PD_API pd_status pd_load_checkpoint(pd_ctx *ctx, const char *dir);

/* Copies the LATEST fp32 parameters of `layer` (master weights) to host_out.  The layer's
 * stage must have a local worker (replica 0 preferred).  count must equal the layer's
 * parameter count (PD_EINVAL otherwise). */
PD_API pd_status pd_get_params(pd_ctx *ctx, int layer, float *host_out, size_t count);

/* Event trace of the last pd_run for the local workers (record_trace >= 1), per worker in
 * issue order == device execution order on that worker's stream. */
typedef struct {
    int16_t worker, stage, replica, kind; /* kind: 'F', 'B', 'U'                         */
    int32_t seq;                          /* index within the worker's sequence          */
    int32_t minibatch;                    /* U on a replicated stage: round index j      */
    int32_t version_in, version_out;      /* weight versions read / written              */
    float start_us, end_us;               /* device times from the run start (record_trace 2) */
} pd_event;

PD_API pd_status pd_get_trace(pd_ctx *ctx, pd_event *out, size_t cap, size_t *written);

/* Version map of the last run: out[s * M + t] = v(s, t), the weight version F(s, t) read;
 * -1 where no local worker of stage s ran minibatch t.  cap >= num_stages * M. */
PD_API pd_status pd_get_version_map(pd_ctx *ctx, int32_t *out, size_t cap);

/* Per-minibatch mean loss of the last run (local last-stage workers; others -> NaN).
 * cap >= M.  This is a small device-to-host read. */
PD_API pd_status pd_get_losses(pd_ctx *ctx, float *out, size_t cap);

#define PD_MAX_LOCAL_WORKERS 64
#define PD_KERNEL_CLASSES 8     /* pd_stats per-class kernel timing */
typedef struct {
    double host_ms;               /* host wall time of the last pd_run                     */
    double device_ms;             /* device span of the last run over the local workers    */
    double bubble;                /* 1 - sum(busy) / (local workers * span)  (record_trace 2) */
    uint64_t kernel_launches;     /* kernels this library launched during the last pd_run  */
    uint64_t bytes_sent;          /* last pd_run: activation + gradient bytes written to other workers */
    int num_local_workers;
    int worker_id[PD_MAX_LOCAL_WORKERS];
    double busy_ms[PD_MAX_LOCAL_WORKERS];  /* sum of F/B op device durations per worker    */
    double span_ms[PD_MAX_LOCAL_WORKERS];  /* first op start to last op end per worker     */
    double run_ms;                /* device time of the last run: max over local workers of
                                     the span between events recorded on the worker's stream
                                     before its first and after its last operation          */
    double kern_ms[PD_KERNEL_CLASSES]; /* record_trace 2: summed device time per kernel class:
                                     0 forward GEMM, 1 dX GEMM, 2 dW GEMM (+fused update),
                                     3 other (bias gradients, pooling, embedding, copies),
                                     4 LSTM wavefront forward, 5 LSTM wavefront backward,
                                     6 softmax-CE, 7 separate optimizer update pass        */
    uint64_t kern_count[PD_KERNEL_CLASSES]; /* launches timed per class                      */
    uint64_t replica_bytes;       /* last pd_run, local workers: peer bytes of the sharded replica
                                     sync -- per round and replica (R-1)/R of the parameters'
                                     fp32 gradients read from the peers, and this replica's 1/R
                                     shard of the new version (fp32 [+ bf16]) stored into each
                                     of the R-1 peers                                        */
} pd_stats;

PD_API pd_status pd_get_stats(pd_ctx *ctx, pd_stats *out);

/* Changes the instrumentation of later pd_run calls: record_trace as in pd_train_cfg;
 * kernel_timing_mask bit c times every kernel of class c with CUDA events on its stream
 * (the PD_KERNEL_CLASSES classes of pd_stats.kern_ms); each timed
 * launch costs two event records, so time only what is needed inside a timed region. */
PD_API pd_status pd_set_timing(pd_ctx *ctx, int record_trace, int kernel_timing_mask);

/* Layer profiling of later pd_run calls (the self-profiler's mechanism, usable on any plan):
 * on = 1 records CUDA events around each layer's share of every F and B op; those ops then
 * run serialised on the worker's stream (no side stream, no CUDA-graph replay), so
 * throughput drops.  pd_get_layer_times returns, for the last run, the mean device seconds
 * per minibatch of each layer's forward / backward over the local workers that ran it
 * (0 for layers without a local worker); count must equal num_layers. */
PD_API pd_status pd_set_layer_profiling(pd_ctx *ctx, int on);
PD_API pd_status pd_get_layer_times(pd_ctx *ctx, double *fwd_s, double *bwd_s, size_t count);

/* Releases everything the context owns.  Safe on NULL. */
PD_API void pd_destroy(pd_ctx *ctx);

/* Static strings, not owned by the caller. */
PD_API const char *pd_strerror(pd_status s);
PD_API const char *pd_last_error(pd_ctx *ctx);

/* In-flight counts k_s for a plan (R2, R19); helper for callers sizing things.  noam as in
 * pd_run.  k_out has num_stages entries. */
PD_API pd_status pd_inflight(const pd_plan_t *plan, int noam, int *k_out);

#ifdef __cplusplus
}
#endif
#endif /* PIPEDREAM_H */
