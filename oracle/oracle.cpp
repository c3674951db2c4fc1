/*
 * oracle.cpp -- TEST INFRASTRUCTURE ONLY.  A plain, slow, single-threaded CPU fp32
 * simulator of PipeDream training (Narayanan et al., SOSP'19, /root/reference/PAPER.md),
 * written step by step from the paper so that a reader can check it by eye.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * legs may load this library.  It shares NO code, header, table or constant with the
 * CUDA product path (paper_conf_sosp_narayananhpsdgg19_b200/csrc); the two agree only
 * through the written parameter/data layout contract in DESIGN.md.
 *
 * What it computes (citations are PAPER.md line numbers, "§" = paper section):
 *   - layer math (linear+ReLU, LSTM, 3x3 conv, 2x2 max-pool, embedding, softmax-CE) as
 *     naive loops, fp32, k-ascending accumulation (the paper trains in fp32, L1591);
 *   - SGD (L1571-1573) and Adam (L1587-1589) updates;
 *   - 1F1B-RR per-worker static op lists (§3.2, reading R3);
 *   - an event-driven executor with explicit per-stage activation/gradient queues,
 *     weight stashing (§3.3), updates applied to the latest weights
 *     (L1341-1353) and replica rounds averaged in replica order (L1345-1347, L1373-1381);
 *   - the GPipe comparison schedule (§5.4): pipeline flushes every D minibatches with the
 *     group's gradients aggregated into one update (L1277-1279);
 *   - an optional timeline (start/end per op, bubble) for Fig. 2/4/8-style pins;
 *   - the §3.1 dynamic-programming partitioner (L899-985) as read in DESIGN.md R10-R16.
 *
 * Parity status: every function below is pinned by tests/test_oracle_*.py (P1-P10 in
 * DESIGN.md).  Learning-curve / accuracy claims of the paper are "parity unpinned" (no
 * datasets, no printed worked example) and are not modelled here.
 */
#include <cmath>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <functional>
#include <vector>

extern "C" {

/* ---- public structs (ctypes mirrors them in oracle/__init__.py) ---- */
enum { ORC_LINEAR = 0, ORC_LSTM = 1, ORC_CONV3X3 = 2, ORC_MAXPOOL2 = 3, ORC_EMBEDDING = 4 };
enum { ORC_ACT_NONE = 0, ORC_ACT_RELU = 1 };
enum { ORC_SGD = 0, ORC_ADAM = 1 };

typedef struct {
    int kind;      /* ORC_* */
    int in, out;   /* features (linear, lstm), channels (conv, pool), vocab/hidden (embedding) */
    int act;       /* ORC_ACT_* (linear, conv) */
    int seq_len;   /* T for sequence models (lstm, embedding, and a linear applied per token) */
    int height, width; /* input spatial size (conv, pool) */
} orc_layer;

typedef struct {
    int worker, stage, replica, seq;
    int kind; /* 'F', 'B', 'U' */
    int minibatch;  /* for U on a replicated stage: round index j */
    int version_in, version_out;
    double start, end;
} orc_event;

}  // extern "C"

namespace {

/* ================================================================== */
/*  Layer shapes                                                       */
/* ================================================================== */

/* rows of the 2-D activation a layer consumes: B for image/MLP layers, T*B for tokens */
long rows_of(const orc_layer &L, int B) { return L.seq_len > 0 ? (long)L.seq_len * B : (long)B; }

long param_count(const orc_layer &L) {
    switch (L.kind) {
    case ORC_LINEAR: return (long)L.out * L.in + L.out;                 /* W[out][in], b[out] */
    case ORC_LSTM: return 4L * L.out * L.in + 4L * L.out * L.out + 8L * L.out; /* Wih,Whh,bih,bhh */
    case ORC_CONV3X3: return (long)L.out * L.in * 9 + L.out;            /* W[co][ci][3][3], b */
    case ORC_MAXPOOL2: return 0;
    case ORC_EMBEDDING: return (long)L.in * L.out;                      /* E[V][H] */
    }
    return -1;
}

/* number of floats of the layer's input / output for a minibatch of B samples */
long in_size(const orc_layer &L, int B) {
    switch (L.kind) {
    case ORC_LINEAR: return rows_of(L, B) * L.in;
    case ORC_LSTM: return (long)L.seq_len * B * L.in;
    case ORC_CONV3X3:
    case ORC_MAXPOOL2: return (long)B * L.height * L.width * L.in;
    case ORC_EMBEDDING: return (long)L.seq_len * B; /* token ids (stored as float-free ints) */
    }
    return -1;
}
long out_size(const orc_layer &L, int B) {
    switch (L.kind) {
    case ORC_LINEAR: return rows_of(L, B) * L.out;
    case ORC_LSTM: return (long)L.seq_len * B * L.out;
    case ORC_CONV3X3: return (long)B * L.height * L.width * L.out;
    case ORC_MAXPOOL2: return (long)B * (L.height / 2) * (L.width / 2) * L.in;
    case ORC_EMBEDDING: return (long)L.seq_len * B * L.out;
    }
    return -1;
}

float sigmoidf_(float x) { return 1.0f / (1.0f + expf(-x)); }

/* ================================================================== */
/*  Layer math: forward                                                */
/* ================================================================== */

/* Linear: y[r][o] = act( (sum_i x[r][i] * W[o][i]) + b[o] ) */
void linear_fwd(const orc_layer &L, int B, const float *p, const float *x, float *y) {
    const float *W = p, *b = p + (long)L.out * L.in;
    long R = rows_of(L, B);
    for (long r = 0; r < R; r++)
        for (int o = 0; o < L.out; o++) {
            float acc = 0.0f;
            for (int i = 0; i < L.in; i++) acc += x[r * L.in + i] * W[(long)o * L.in + i];
            float z = acc + b[o];
            y[r * L.out + o] = (L.act == ORC_ACT_RELU && z < 0.0f) ? 0.0f : z;
        }
}

/* LSTM (PyTorch form, gate order i,f,g,o; h0 = c0 = 0).  x, y time-major [T][B][feat].
 * If hs/cs/gs are given they receive h_t, c_t and the post-nonlinearity gates per step. */
void lstm_fwd(const orc_layer &L, int B, const float *p, const float *x, float *y,
              float *hs = nullptr, float *cs = nullptr, float *gs = nullptr) {
    const int H = L.out, I = L.in, T = L.seq_len;
    const float *Wih = p, *Whh = Wih + 4L * H * I, *bih = Whh + 4L * H * H, *bhh = bih + 4L * H;
    std::vector<float> h((long)B * H, 0.0f), c((long)B * H, 0.0f), g(4L * H);
    for (int t = 0; t < T; t++) {
        std::vector<float> hn((long)B * H), cn((long)B * H);
        for (int b = 0; b < B; b++) {
            const float *xt = x + ((long)t * B + b) * I;
            for (int k = 0; k < 4 * H; k++) {
                float ax = 0.0f;
                for (int i = 0; i < I; i++) ax += xt[i] * Wih[(long)k * I + i];
                float ah = 0.0f;
                for (int j = 0; j < H; j++) ah += h[(long)b * H + j] * Whh[(long)k * H + j];
                float a = ax + bih[k] + ah + bhh[k];
                int gate = k / H;
                g[k] = (gate == 2) ? tanhf(a) : sigmoidf_(a);
            }
            for (int j = 0; j < H; j++) {
                float ig = g[j], fg = g[H + j], gg = g[2 * H + j], og = g[3 * H + j];
                float cv = fg * c[(long)b * H + j] + ig * gg;
                cn[(long)b * H + j] = cv;
                hn[(long)b * H + j] = og * tanhf(cv);
            }
            if (gs) memcpy(gs + ((long)t * B + b) * 4 * H, g.data(), sizeof(float) * 4 * H);
        }
        h = hn;
        c = cn;
        memcpy(y + (long)t * B * H, h.data(), sizeof(float) * B * H);
        if (hs) memcpy(hs + (long)t * B * H, h.data(), sizeof(float) * B * H);
        if (cs) memcpy(cs + (long)t * B * H, c.data(), sizeof(float) * B * H);
    }
}

/* 3x3 conv, stride 1, zero pad 1, NHWC.  y[b][h][w][co] = act(sum_{ci,kh,kw} x*W + b) */
void conv_fwd(const orc_layer &L, int B, const float *p, const float *x, float *y) {
    const int H = L.height, Wd = L.width, Ci = L.in, Co = L.out;
    const float *W = p, *bias = p + (long)Co * Ci * 9;
    for (int b = 0; b < B; b++)
        for (int h = 0; h < H; h++)
            for (int w = 0; w < Wd; w++)
                for (int co = 0; co < Co; co++) {
                    float acc = 0.0f;
                    for (int ci = 0; ci < Ci; ci++)
                        for (int kh = 0; kh < 3; kh++)
                            for (int kw = 0; kw < 3; kw++) {
                                int ih = h + kh - 1, iw = w + kw - 1;
                                if (ih < 0 || ih >= H || iw < 0 || iw >= Wd) continue;
                                acc += x[(((long)b * H + ih) * Wd + iw) * Ci + ci] *
                                       W[(((long)co * Ci + ci) * 3 + kh) * 3 + kw];
                            }
                    float z = acc + bias[co];
                    y[(((long)b * H + h) * Wd + w) * Co + co] = (L.act == ORC_ACT_RELU && z < 0.0f) ? 0.0f : z;
                }
}

/* 2x2 max-pool stride 2, NHWC; the first maximum in (dh, dw) scan order wins ties */
void pool_fwd(const orc_layer &L, int B, const float *x, float *y, int *arg = nullptr) {
    const int H = L.height, Wd = L.width, C = L.in, Ho = H / 2, Wo = Wd / 2;
    for (int b = 0; b < B; b++)
        for (int h = 0; h < Ho; h++)
            for (int w = 0; w < Wo; w++)
                for (int c = 0; c < C; c++) {
                    float best = 0.0f;
                    long bi = -1;
                    for (int dh = 0; dh < 2; dh++)
                        for (int dw = 0; dw < 2; dw++) {
                            long idx = (((long)b * H + 2 * h + dh) * Wd + 2 * w + dw) * C + c;
                            if (bi < 0 || x[idx] > best) { best = x[idx]; bi = idx; }
                        }
                    long o = (((long)b * Ho + h) * Wo + w) * C + c;
                    y[o] = best;
                    if (arg) arg[o] = (int)bi;
                }
}

/* Embedding: y[t][b][:] = E[tok[t][b]][:] */
void emb_fwd(const orc_layer &L, int B, const float *p, const int *tok, float *y) {
    long R = (long)L.seq_len * B;
    for (long r = 0; r < R; r++) memcpy(y + r * L.out, p + (long)tok[r] * L.out, sizeof(float) * L.out);
}

void layer_fwd(const orc_layer &L, int B, const float *p, const float *x, const int *tok, float *y) {
    switch (L.kind) {
    case ORC_LINEAR: linear_fwd(L, B, p, x, y); break;
    case ORC_LSTM: lstm_fwd(L, B, p, x, y); break;
    case ORC_CONV3X3: conv_fwd(L, B, p, x, y); break;
    case ORC_MAXPOOL2: pool_fwd(L, B, x, y); break;
    case ORC_EMBEDDING: emb_fwd(L, B, p, tok, y); break;
    }
}

/* ================================================================== */
/*  Layer math: backward.  dy is the gradient w.r.t. the layer output  */
/*  (post-activation).  dx may be null (first layer of stage 0 skips   */
/*  it).  dp receives the parameter gradient (overwritten).  The      */
/*  forward internals are recomputed from the saved input x and the    */
/*  stashed weights p (deterministic, so identical to saving them).    */
/* ================================================================== */

void linear_bwd(const orc_layer &L, int B, const float *p, const float *x, const float *dy, float *dx, float *dp) {
    const float *W = p;
    long R = rows_of(L, B);
    std::vector<float> y(R * L.out), dz(R * L.out);
    linear_fwd(L, B, p, x, y.data());
    for (long k = 0; k < R * L.out; k++) dz[k] = (L.act == ORC_ACT_RELU && !(y[k] > 0.0f)) ? 0.0f : dy[k];
    if (dx)
        for (long r = 0; r < R; r++)
            for (int i = 0; i < L.in; i++) {
                float acc = 0.0f;
                for (int o = 0; o < L.out; o++) acc += dz[r * L.out + o] * W[(long)o * L.in + i];
                dx[r * L.in + i] = acc;
            }
    float *dW = dp, *db = dp + (long)L.out * L.in;
    for (int o = 0; o < L.out; o++) {
        for (int i = 0; i < L.in; i++) {
            float acc = 0.0f;
            for (long r = 0; r < R; r++) acc += dz[r * L.out + o] * x[r * L.in + i];
            dW[(long)o * L.in + i] = acc;
        }
        float acc = 0.0f;
        for (long r = 0; r < R; r++) acc += dz[r * L.out + o];
        db[o] = acc;
    }
}

/* LSTM backpropagation through time (standard derivation of the forward above). */
void lstm_bwd(const orc_layer &L, int B, const float *p, const float *x, const float *dy, float *dx, float *dp) {
    const int H = L.out, I = L.in, T = L.seq_len;
    const float *Wih = p, *Whh = Wih + 4L * H * I;
    std::vector<float> y((long)T * B * H), hs((long)T * B * H), cs((long)T * B * H), gs((long)T * B * 4 * H);
    lstm_fwd(L, B, p, x, y.data(), hs.data(), cs.data(), gs.data());
    float *dWih = dp, *dWhh = dWih + 4L * H * I, *dbih = dWhh + 4L * H * H, *dbhh = dbih + 4L * H;
    memset(dp, 0, sizeof(float) * param_count(L));
    std::vector<float> dh((long)B * H, 0.0f), dc((long)B * H, 0.0f), da((long)B * 4 * H);
    for (int t = T - 1; t >= 0; t--) {
        for (int b = 0; b < B; b++) {
            const float *g = gs.data() + ((long)t * B + b) * 4 * H;
            for (int j = 0; j < H; j++) {
                long bj = (long)b * H + j;
                float c = cs[(long)t * B * H + bj];
                float cprev = t > 0 ? cs[(long)(t - 1) * B * H + bj] : 0.0f;
                float ig = g[j], fg = g[H + j], gg = g[2 * H + j], og = g[3 * H + j];
                float tc = tanhf(c);
                float dht = dy[(long)t * B * H + bj] + dh[bj];
                float dog = dht * tc;
                float dct = dht * og * (1.0f - tc * tc) + dc[bj];
                float dig = dct * gg, dgg = dct * ig, dfg = dct * cprev;
                dc[bj] = dct * fg;
                float *a = da.data() + (long)b * 4 * H;
                a[j] = dig * ig * (1.0f - ig);
                a[H + j] = dfg * fg * (1.0f - fg);
                a[2 * H + j] = dgg * (1.0f - gg * gg);
                a[3 * H + j] = dog * og * (1.0f - og);
            }
        }
        /* parameter gradients, accumulated over t descending then b ascending */
        for (int k = 0; k < 4 * H; k++) {
            for (int b = 0; b < B; b++) {
                float a = da[(long)b * 4 * H + k];
                const float *xt = x + ((long)t * B + b) * I;
                for (int i = 0; i < I; i++) dWih[(long)k * I + i] += a * xt[i];
                if (t > 0) {
                    const float *hp = hs.data() + ((long)(t - 1) * B + b) * H;
                    for (int j = 0; j < H; j++) dWhh[(long)k * H + j] += a * hp[j];
                }
                dbih[k] += a;
                dbhh[k] += a;
            }
        }
        for (int b = 0; b < B; b++) {
            const float *a = da.data() + (long)b * 4 * H;
            if (dx)
                for (int i = 0; i < I; i++) {
                    float acc = 0.0f;
                    for (int k = 0; k < 4 * H; k++) acc += a[k] * Wih[(long)k * I + i];
                    dx[((long)t * B + b) * I + i] = acc;
                }
            for (int j = 0; j < H; j++) {
                float acc = 0.0f;
                for (int k = 0; k < 4 * H; k++) acc += a[k] * Whh[(long)k * H + j];
                dh[(long)b * H + j] = acc;
            }
        }
    }
}

void conv_bwd(const orc_layer &L, int B, const float *p, const float *x, const float *dy, float *dx, float *dp) {
    const int H = L.height, Wd = L.width, Ci = L.in, Co = L.out;
    const float *W = p;
    long n = out_size(L, B);
    std::vector<float> y(n), dz(n);
    conv_fwd(L, B, p, x, y.data());
    for (long k = 0; k < n; k++) dz[k] = (L.act == ORC_ACT_RELU && !(y[k] > 0.0f)) ? 0.0f : dy[k];
    if (dx)
        for (int b = 0; b < B; b++)
            for (int ih = 0; ih < H; ih++)
                for (int iw = 0; iw < Wd; iw++)
                    for (int ci = 0; ci < Ci; ci++) {
                        float acc = 0.0f;
                        for (int co = 0; co < Co; co++)
                            for (int kh = 0; kh < 3; kh++)
                                for (int kw = 0; kw < 3; kw++) {
                                    int h = ih - kh + 1, w = iw - kw + 1;
                                    if (h < 0 || h >= H || w < 0 || w >= Wd) continue;
                                    acc += dz[(((long)b * H + h) * Wd + w) * Co + co] *
                                           W[(((long)co * Ci + ci) * 3 + kh) * 3 + kw];
                                }
                        dx[(((long)b * H + ih) * Wd + iw) * Ci + ci] = acc;
                    }
    float *dW = dp, *db = dp + (long)Co * Ci * 9;
    for (int co = 0; co < Co; co++) {
        for (int ci = 0; ci < Ci; ci++)
            for (int kh = 0; kh < 3; kh++)
                for (int kw = 0; kw < 3; kw++) {
                    float acc = 0.0f;
                    for (int b = 0; b < B; b++)
                        for (int h = 0; h < H; h++)
                            for (int w = 0; w < Wd; w++) {
                                int ih = h + kh - 1, iw = w + kw - 1;
                                if (ih < 0 || ih >= H || iw < 0 || iw >= Wd) continue;
                                acc += dz[(((long)b * H + h) * Wd + w) * Co + co] *
                                       x[(((long)b * H + ih) * Wd + iw) * Ci + ci];
                            }
                    dW[(((long)co * Ci + ci) * 3 + kh) * 3 + kw] = acc;
                }
        float acc = 0.0f;
        for (int b = 0; b < B; b++)
            for (int h = 0; h < H; h++)
                for (int w = 0; w < Wd; w++) acc += dz[(((long)b * H + h) * Wd + w) * Co + co];
        db[co] = acc;
    }
}

void pool_bwd(const orc_layer &L, int B, const float *x, const float *dy, float *dx) {
    long n = out_size(L, B);
    std::vector<float> y(n);
    std::vector<int> arg(n);
    pool_fwd(L, B, x, y.data(), arg.data());
    if (!dx) return;
    memset(dx, 0, sizeof(float) * in_size(L, B));
    for (long o = 0; o < n; o++) dx[arg[o]] += dy[o];
}

void emb_bwd(const orc_layer &L, int B, const int *tok, const float *dy, float *dp) {
    memset(dp, 0, sizeof(float) * param_count(L));
    long R = (long)L.seq_len * B;
    for (long r = 0; r < R; r++)
        for (int j = 0; j < L.out; j++) dp[(long)tok[r] * L.out + j] += dy[r * L.out + j];
}

void layer_bwd(const orc_layer &L, int B, const float *p, const float *x, const int *tok, const float *dy,
               float *dx, float *dp) {
    switch (L.kind) {
    case ORC_LINEAR: linear_bwd(L, B, p, x, dy, dx, dp); break;
    case ORC_LSTM: lstm_bwd(L, B, p, x, dy, dx, dp); break;
    case ORC_CONV3X3: conv_bwd(L, B, p, x, dy, dx, dp); break;
    case ORC_MAXPOOL2: pool_bwd(L, B, x, dy, dx); break;
    case ORC_EMBEDDING: emb_bwd(L, B, tok, dy, dp); break;
    }
}

/* Softmax cross-entropy, mean over rows (L1217: gradient averaged over the minibatch;
 * DESIGN.md R8: mean over B*T tokens for sequence models). */
float softmax_ce(const float *z, const int *label, long R, int C, float *dz) {
    double total = 0.0; /* the loss value is reported only; it does not feed the math */
    for (long r = 0; r < R; r++) {
        const float *zr = z + r * C;
        float m = zr[0];
        for (int c = 1; c < C; c++) m = zr[c] > m ? zr[c] : m;
        float s = 0.0f;
        for (int c = 0; c < C; c++) s += expf(zr[c] - m);
        float lse = m + logf(s);
        total += (double)(lse - zr[label[r]]);
        if (dz)
            for (int c = 0; c < C; c++) {
                float sm = expf(zr[c] - m) / s;
                dz[r * C + c] = (sm - (c == label[r] ? 1.0f : 0.0f)) / (float)R;
            }
    }
    return (float)(total / (double)R);
}

/* ================================================================== */
/*  Optimizers (R9).  Applied to the LATEST weights          */
/*  (L1341-1345).  step = number of updates applied so far + 1.        */
/* ================================================================== */
struct OptCfg { int kind; float lr, b1, b2, eps; };

void apply_update(const OptCfg &o, float *w, const float *g, float *m, float *v, long n, int step) {
    if (o.kind == ORC_SGD) {
        for (long k = 0; k < n; k++) w[k] = w[k] - o.lr * g[k];
        return;
    }
    float bc1 = 1.0f - powf(o.b1, (float)step), bc2 = 1.0f - powf(o.b2, (float)step);
    for (long k = 0; k < n; k++) {
        m[k] = o.b1 * m[k] + (1.0f - o.b1) * g[k];
        v[k] = o.b2 * v[k] + (1.0f - o.b2) * g[k] * g[k];
        float mh = m[k] / bc1, vh = v[k] / bc2;
        w[k] = w[k] - o.lr * mh / (sqrtf(vh) + o.eps);
    }
}

/* ================================================================== */
/*  The 1F1B-RR simulator                                              */
/* ================================================================== */

struct Op { int kind; int t; int round; };

struct Worker {
    int id, stage, replica;
    std::vector<Op> ops;
    size_t pc = 0;
    int version = 0;               /* number of updates applied (replicated: rounds) */
    std::map<int, std::vector<float>> versions; /* stashed versions still referenced */
    std::map<int, int> refcount;   /* version -> pending backward passes using it   */
    std::vector<float> m, v;       /* Adam state (not versioned, R9)                 */
    std::map<int, int> fwd_version;               /* t -> version used in F(s,t)     */
    std::map<int, std::vector<std::vector<float>>> saved; /* t -> per-layer inputs   */
    std::vector<float> grad;       /* gradient of the last backward (all stage params) */
    int last_b_t = -1;
    int b_done = 0;                /* backward passes completed (replicated: round count) */
    double free_at = 0.0;
    int seq = 0;
    int f_done = 0;                /* forwards completed                                     */
    int last_tag = 0;              /* version used by the latest forward (vertical sync)     */
    int max_live = 1;              /* widest version window held (pin P10)                   */
    std::vector<std::vector<float>> group_g; /* GPipe: the gradients of the current group, in t order */
};

struct Sim {
    const orc_layer *layers;
    int n_layers, n_stages, B, M, depth;
    std::vector<int> first, last, R, k;
    std::vector<long> poff; /* parameter offset of each layer in the flat params array */
    long ptotal = 0;
    OptCfg opt;
    bool math, stash;
    bool vsync;             /* vertical sync (§3.3): every stage uses the tag version */
    bool gpipe;             /* GPipe-style flush (§5.4) with gradient aggregation (L1277-1279) */
    int group;              /* GPipe: minibatches per flush group (the pipeline depth D)          */
    std::map<std::pair<int, int>, int> act_tag; /* (stage, t) -> version tag travelling with the activation */
    const float *inputs; const int *tokens, *labels; int n_data;
    const double *ftime, *btime;
    std::vector<Worker> W;
    std::vector<int> wbase; /* first worker id of each stage */
    /* queues: activation into stage s for minibatch t, gradient into stage s for t */
    std::map<std::pair<int, int>, std::vector<float>> act_q, grad_q;
    std::map<std::pair<int, int>, double> act_t, grad_t;
    /* replicated rounds: (stage, j) -> per-replica grads and ready times */
    std::map<std::pair<int, int>, std::vector<std::vector<float>>> round_g;
    std::map<std::pair<int, int>, std::vector<double>> round_t;
    std::map<std::pair<int, int>, std::vector<float>> round_mean;
    std::vector<orc_event> ev;
    std::vector<int> vmap;
    std::vector<float> losses;

    long stage_params(int s) const { return poff[last[s] + 1] - poff[first[s]]; }
};

long sample_in_size(const orc_layer &L) { return in_size(L, 1); }

/* Per-worker static op list (§3.2, R3): F(t_0..t_{k-1}), then (B(t_j) U F(t_{j+k}))*,
 * then (B U)* for the remaining minibatches.  U immediately follows B (L237-241). */
void build_ops(Sim &S, Worker &w) {
    int s = w.stage, Rs = S.R[s];
    if (S.gpipe) {
        /* GPipe (R27): minibatches in groups of D; every stage but the last forwards
         * the whole group, then runs its backwards in t order; the last stage runs F(t) B(t)
         * back to back (its backward starts immediately, L719-721); one U per group applies
         * the aggregated gradient (the flush).  Op.round = group index. */
        for (int g = 0; g * S.group < S.M; g++) {
            int t0 = g * S.group, t1 = t0 + S.group;
            if (s + 1 < S.n_stages) {
                for (int t = t0; t < t1; t++) w.ops.push_back({'F', t, g});
                for (int t = t0; t < t1; t++) w.ops.push_back({'B', t, g});
            } else {
                for (int t = t0; t < t1; t++) { w.ops.push_back({'F', t, g}); w.ops.push_back({'B', t, g}); }
            }
            w.ops.push_back({'U', t1 - 1, g});
        }
        return;
    }
    std::vector<int> ts;
    for (int t = w.replica; t < S.M; t += Rs) ts.push_back(t);
    int Mr = (int)ts.size();
    int k = S.k[s] < Mr ? S.k[s] : Mr;
    for (int j = 0; j < k; j++) w.ops.push_back({'F', ts[j], -1});
    for (int j = 0; j < Mr; j++) {
        w.ops.push_back({'B', ts[j], j});
        w.ops.push_back({'U', ts[j], j});
        if (j + k < Mr) w.ops.push_back({'F', ts[j + k], -1});
    }
}

void emit(Sim &S, Worker &w, int kind, int t, int vin, int vout, double st, double en) {
    orc_event e;
    e.worker = w.id; e.stage = w.stage; e.replica = w.replica; e.seq = w.seq++;
    e.kind = kind; e.minibatch = t; e.version_in = vin; e.version_out = vout; e.start = st; e.end = en;
    S.ev.push_back(e);
}

/* forward of stage s on minibatch t with weights `params` (flat, stage-local) */
void stage_forward(Sim &S, Worker &w, int t, const float *params, const std::vector<float> &input,
                   std::vector<std::vector<float>> &saved, std::vector<float> &out) {
    int s = w.stage, d = t % S.n_data;
    std::vector<float> x = input;
    for (int l = S.first[s]; l <= S.last[s]; l++) {
        const orc_layer &L = S.layers[l];
        const float *p = params + (S.poff[l] - S.poff[S.first[s]]);
        saved.push_back(x);
        std::vector<float> y(out_size(L, S.B));
        const int *tok = (L.kind == ORC_EMBEDDING) ? S.tokens + (long)d * L.seq_len * S.B : nullptr;
        layer_fwd(L, S.B, p, x.data(), tok, y.data());
        x.swap(y);
    }
    out.swap(x);
}

bool ready(Sim &S, Worker &w, const Op &op) {
    int s = w.stage;
    if (op.kind == 'F') return s == 0 || S.act_q.count({s, op.t});
    if (op.kind == 'B') return s == S.n_stages - 1 || S.grad_q.count({s, op.t});
    /* U: replicated stages need every replica's op.round-th backward (L1345-1347) */
    if (S.R[s] == 1) return true;
    auto it = S.round_t.find({s, op.round});
    if (it == S.round_t.end()) return false;
    for (double x : it->second) if (x < 0) return false;
    return true;
}

void exec(Sim &S, Worker &w, const Op &op) {
    int s = w.stage, t = op.t;
    long np = S.stage_params(s);
    if (op.kind == 'F') {
        /* F(s,t): latest version, stash it (L1145-1161).  Vertical sync: the input stage tags
         * t with its latest version and every later stage uses its own stashed weights of
         * that version -- the tag travels with the activation (L1180-1186) */
        int v = w.version;
        if (S.vsync) {
            if (s > 0) v = S.act_tag[{s, t}];
            if (s + 1 < S.n_stages) S.act_tag[{s + 1, t}] = v;
            if (s > 0) S.act_tag.erase({s, t});
        }
        w.f_done++;
        w.last_tag = v;
        double st = w.free_at;
        if (s > 0) st = st > S.act_t[{s, t}] ? st : S.act_t[{s, t}];
        double en = st + (S.ftime ? S.ftime[s] : 0.0);
        w.free_at = en;
        w.fwd_version[t] = v;
        w.refcount[v]++;
        S.vmap[(long)s * S.M + t] = v;
        emit(S, w, 'F', t, v, v, st, en);
        if (S.math) {
            std::vector<float> input;
            if (s == 0) {
                const orc_layer &L0 = S.layers[0];
                int d = t % S.n_data;
                if (L0.kind != ORC_EMBEDDING) {
                    long n = sample_in_size(L0) * S.B;
                    input.assign(S.inputs + (long)d * n, S.inputs + (long)d * n + n);
                }
            } else {
                input = S.act_q[{s, t}];
            }
            std::vector<std::vector<float>> saved;
            std::vector<float> out;
            stage_forward(S, w, t, w.versions[v].data(), input, saved, out);
            w.saved[t] = saved;
            if (s + 1 < S.n_stages) {
                S.act_q[{s + 1, t}] = out;
            } else {
                /* last stage: loss and dlogits; its backward follows immediately (L719-721) */
                const orc_layer &LL = S.layers[S.n_layers - 1];
                long rows = rows_of(LL, S.B);
                int C = LL.kind == ORC_LINEAR ? LL.out : LL.out;
                std::vector<float> dz(out.size());
                S.losses[t] = softmax_ce(out.data(), S.labels + (long)(t % S.n_data) * rows, rows, C, dz.data());
                S.grad_q[{s, t}] = dz;
            }
        }
        if (s + 1 < S.n_stages) S.act_t[{s + 1, t}] = en;
        else S.grad_t[{s, t}] = en;
        if (!S.math && s + 1 < S.n_stages) S.act_q[{s + 1, t}] = {};
        if (!S.math && s + 1 == S.n_stages) S.grad_q[{s, t}] = {};
        if (s > 0) { S.act_q.erase({s, t}); }
        return;
    }
    if (op.kind == 'B') {
        /* B(s,t): stashed version (or latest for the negative control) */
        int v = w.fwd_version[t];
        int vuse = S.stash ? v : w.version;
        double st = w.free_at;
        double gt = S.grad_t[{s, t}];
        st = st > gt ? st : gt;
        double en = st + (S.btime ? S.btime[s] : 0.0);
        w.free_at = en;
        emit(S, w, 'B', t, v, v, st, en);
        if (S.math) {
            const float *params = w.versions[S.stash ? v : w.version].data();
            (void)vuse;
            std::vector<float> dy = S.grad_q[{s, t}];
            auto &saved = w.saved[t];
            w.grad.assign(np, 0.0f);
            for (int l = S.last[s]; l >= S.first[s]; l--) {
                const orc_layer &L = S.layers[l];
                long off = S.poff[l] - S.poff[S.first[s]];
                const float *x = saved[l - S.first[s]].data();
                const int *tok = (L.kind == ORC_EMBEDDING) ? S.tokens + (long)(t % S.n_data) * L.seq_len * S.B : nullptr;
                bool need_dx = !(s == 0 && l == 0); /* stage 0 skips dX of its first layer */
                std::vector<float> dx(need_dx ? in_size(L, S.B) : 0);
                layer_bwd(L, S.B, params + off, x, tok, dy.data(), need_dx ? dx.data() : nullptr, w.grad.data() + off);
                dy.swap(dx);
            }
            if (s > 0) S.grad_q[{s - 1, t}] = dy;
            w.saved.erase(t);
        } else if (s > 0) {
            S.grad_q[{s - 1, t}] = {};
        }
        if (s > 0) S.grad_t[{s - 1, t}] = en;
        S.grad_q.erase({s, t});
        w.last_b_t = t;
        if (S.gpipe && S.math) w.group_g.push_back(w.grad);
        if (S.R[s] > 1) {
            auto key = std::make_pair(s, op.round);
            if (!S.round_t.count(key)) {
                S.round_t[key] = std::vector<double>(S.R[s], -1.0);
                S.round_g[key] = std::vector<std::vector<float>>(S.R[s]);
            }
            S.round_t[key][w.replica] = en;
            S.round_g[key][w.replica] = w.grad;
        }
        return;
    }
    /* U: apply the update to the latest weights, creating version+1 (L1341-1353) */
    int vin = w.version;
    double st = w.free_at;
    const float *g = nullptr;
    std::vector<float> mean;
    int ev_t = t;
    if (S.R[s] > 1) {
        auto key = std::make_pair(s, op.round);
        for (double x : S.round_t[key]) st = st > x ? st : x;
        if (S.math) {
            if (!S.round_mean.count(key)) {
                /* mean = (sum over replicas in r order) * (1/R)  (R7) */
                std::vector<float> acc(np, 0.0f);
                for (int r = 0; r < S.R[s]; r++)
                    for (long k2 = 0; k2 < np; k2++) acc[k2] += S.round_g[key][r][k2];
                float inv = 1.0f / (float)S.R[s];
                for (long k2 = 0; k2 < np; k2++) acc[k2] = acc[k2] * inv;
                S.round_mean[key] = acc;
            }
            g = S.round_mean[key].data();
        }
        ev_t = op.round;
    } else if (S.gpipe) {
        /* gradient aggregation (L1277-1279): the group's D gradients added in t order into one
         * buffer, times 1/D -- the mean over the group, so that a flush group of D minibatches
         * of B samples is one SGD step on D*B samples (R27) */
        if (S.math) {
            mean.assign(np, 0.0f);
            for (auto &gt : w.group_g)
                for (long k2 = 0; k2 < np; k2++) mean[k2] += gt[k2];
            float inv = 1.0f / (float)w.group_g.size();
            for (long k2 = 0; k2 < np; k2++) mean[k2] = mean[k2] * inv;
            g = mean.data();
            w.group_g.clear();
        }
        ev_t = op.round;
    } else if (S.math) {
        g = w.grad.data();
    }
    w.free_at = st;
    if (S.math) {
        std::vector<float> nw = w.versions[vin];
        apply_update(S.opt, nw.data(), g, w.m.data(), w.v.data(), np, vin + 1);
        w.versions[vin + 1] = nw;
    } else {
        w.versions[vin + 1] = {};
    }
    w.version = vin + 1;
    emit(S, w, 'U', ev_t, vin, vin + 1, st, st);

    /* the stashed version of the backward just applied is released; a version is discarded
     * once no pending backward references it and it is not the latest (L1349-1353) */
    if (S.gpipe) {
        /* the flush: every minibatch of the group has finished its backward */
        for (int t2 = op.round * S.group; t2 <= t; t2++) {
            w.refcount[w.fwd_version[t2]]--;
            w.fwd_version.erase(t2);
        }
    } else {
        int vb = w.fwd_version[t];
        w.refcount[vb]--;
        w.fwd_version.erase(t);
    }
    /* vertical sync: a minibatch not yet forwarded here carries a tag >= the tag of the
     * last one forwarded here (the input stage's version only grows and it forwards in t
     * order; straight pipelines), so versions from that tag on are kept */
    int keep_from = 1 << 30;
    if (S.vsync && w.f_done < S.M) keep_from = w.last_tag;
    for (auto it = w.versions.begin(); it != w.versions.end();) {
        int ver = it->first;
        if (ver != w.version && w.refcount[ver] <= 0 && ver < keep_from) it = w.versions.erase(it);
        else ++it;
    }
    /* window of versions held after the update: a ring indexed by version mod depth needs
     * depth >= this span (the consumed version's storage receives the new one) */
    int span = w.versions.rbegin()->first - w.versions.begin()->first + 1;
    if (span > w.max_live) w.max_live = span;
    if (S.R[s] > 1) {
        /* free round buffers once every replica has applied it */
        bool all = true;
        for (int r = 0; r < S.R[s]; r++) if (S.W[S.wbase[s] + r].version <= op.round) all = false;
        if (all) {
            auto key = std::make_pair(s, op.round);
            S.round_g.erase(key); S.round_mean.erase(key);
        }
    }
}

int ceil_div(int a, int b) { return (a + b - 1) / b; }

}  // namespace

extern "C" {

long orc_param_count(const orc_layer *L) { return param_count(*L); }
long orc_in_size(const orc_layer *L, int B) { return in_size(*L, B); }
long orc_out_size(const orc_layer *L, int B) { return out_size(*L, B); }

/* single-layer entry points used by the layer-math pins (P9) */
int orc_layer_forward(const orc_layer *L, int B, const float *params, const float *x, const int *tok, float *y) {
    layer_fwd(*L, B, params, x, tok, y);
    return 0;
}
int orc_layer_backward(const orc_layer *L, int B, const float *params, const float *x, const int *tok,
                       const float *dy, float *dx, float *dparams) {
    layer_bwd(*L, B, params, x, tok, dy, dx, dparams);
    return 0;
}
float orc_softmax_ce(const float *logits, const int *labels, long rows, int C, float *dlogits) {
    return softmax_ce(logits, labels, rows, C, dlogits);
}
void orc_update(int kind, float lr, float b1, float b2, float eps, float *w, const float *g, float *m, float *v,
                long n, int step) {
    OptCfg o{kind, lr, b1, b2, eps};
    apply_update(o, w, g, m, v, n, step);
}

/* In-flight count per stage (R2, R19).  k_s = ceil(W_{>=s} / R_s); NOAM = k_0
 * (L1021, ceiling per R1).  A depth override D (straight plans only) gives
 * k_s = max(1, D - s) for s < n-1 and k_{n-1} = 1. */
int orc_inflight(const int *R, int n, int depth, int *k_out) {
    int straight = 1;
    for (int s = 0; s < n; s++) if (R[s] != 1) straight = 0;
    if (depth > 0 && !straight) return -1;
    for (int s = 0; s < n; s++) {
        if (depth > 0) {
            int ks = depth - s;
            k_out[s] = (s == n - 1) ? 1 : (ks > 1 ? ks : 1);
        } else {
            int wge = 0;
            for (int q = s; q < n; q++) wge += R[q];
            k_out[s] = ceil_div(wge, R[s]);
        }
    }
    return 0;
}

/*
 * Run PipeDream 1F1B-RR with weight stashing.
 *   stage_last[s]  : index of the last layer of stage s (stages are contiguous from layer 0)
 *   replicas[s]    : R_s
 *   depth          : 0 => default in-flight counts (NOAM), else the R19 override
 *   mode bit0      : 1 = do the math, 0 = schedule only
 *   mode bit1      : 1 = disable weight stashing (negative control; backward uses latest)
 *   mode bit2      : 1 = vertical sync (§3.3; straight pipelines only)
 *   mode bit3      : 1 = GPipe-style flush schedule with gradient aggregation (§5.4,
 *                    L1277-1279; R27): groups of D = depth (0 => n) minibatches, one
 *                    update per group with the mean of the group's gradients; straight only
 *   inputs/tokens/labels: n_data minibatches, minibatch t uses data t mod n_data
 *   params         : in = initial flat params (layer order), out = final latest params
 *                    (replica 0 of every stage; replicas are identical by construction)
 *   fwd/bwd_time   : per-stage durations for the timeline (may be NULL => 0)
 *   max_live       : per stage, the widest window (newest - oldest + 1) of weight versions a
 *                    worker held after an update (may be NULL)
 * Returns 0, or -1 invalid, -2 deadlock, -3 event buffer too small.
 */
int orc_run(const orc_layer *layers, int n_layers, const int *stage_last, const int *replicas, int n_stages,
            int depth, int B, int M, int opt_kind, float lr, float b1, float b2, float eps, int mode,
            const float *inputs, const int *tokens, const int *labels, int n_data, float *params,
            const double *fwd_time, const double *bwd_time, orc_event *events, int events_cap, int *n_events,
            int *version_map, float *losses, double *makespan, double *bubble, int *max_live) {
    Sim S;
    S.layers = layers; S.n_layers = n_layers; S.n_stages = n_stages; S.B = B; S.M = M; S.depth = depth;
    S.opt = OptCfg{opt_kind, lr, b1, b2, eps};
    S.math = (mode & 1) != 0; S.stash = (mode & 2) == 0; S.vsync = (mode & 4) != 0; S.gpipe = (mode & 8) != 0;
    S.inputs = inputs; S.tokens = tokens; S.labels = labels; S.n_data = n_data > 0 ? n_data : 1;
    S.ftime = fwd_time; S.btime = bwd_time;
    if (n_stages < 1 || stage_last[n_stages - 1] != n_layers - 1) return -1;
    for (int s = 0; s < n_stages; s++) {
        S.first.push_back(s == 0 ? 0 : stage_last[s - 1] + 1);
        S.last.push_back(stage_last[s]);
        if (S.last[s] < S.first[s] || replicas[s] < 1) return -1;
        if (M % replicas[s] != 0) return -1;
        S.R.push_back(replicas[s]);
    }
    if (S.vsync) {
        if (!S.stash) return -1;
        for (int s = 0; s < n_stages; s++) if (S.R[s] != 1) return -1; /* straight pipelines only */
    }
    S.k.assign(n_stages, 0);
    if (S.gpipe) {
        /* GPipe: straight plans, no vertical sync; group D = depth, or NOAM = n when depth = 0
         * (the paper's "pipeline depth equivalent to NOAM", L1955-1958); M a multiple of D */
        if (S.vsync) return -1;
        for (int s = 0; s < n_stages; s++) if (S.R[s] != 1) return -1;
        S.group = depth > 0 ? depth : n_stages;
        if (M % S.group != 0) return -1;
        depth = 0;
    }
    if (orc_inflight(replicas, n_stages, depth, S.k.data()) != 0) return -1;
    S.poff.assign(n_layers + 1, 0);
    for (int l = 0; l < n_layers; l++) S.poff[l + 1] = S.poff[l] + param_count(layers[l]);
    S.ptotal = S.poff[n_layers];
    S.vmap.assign((long)n_stages * M, -1);
    S.losses.assign(M, 0.0f);
    int id = 0;
    for (int s = 0; s < n_stages; s++) {
        S.wbase.push_back(id);
        for (int r = 0; r < S.R[s]; r++) {
            Worker w;
            w.id = id++; w.stage = s; w.replica = r;
            long np = S.stage_params(s);
            if (S.math) {
                w.versions[0].assign(params + S.poff[S.first[s]], params + S.poff[S.first[s]] + np);
                if (opt_kind == ORC_ADAM) { w.m.assign(np, 0.0f); w.v.assign(np, 0.0f); }
            } else {
                w.versions[0] = {};
            }
            build_ops(S, w);
            S.W.push_back(w);
        }
    }
    /* event-driven execution: each worker pops its next op when its inputs are present */
    for (;;) {
        bool progress = false, done = true;
        for (auto &w : S.W) {
            while (w.pc < w.ops.size() && ready(S, w, w.ops[w.pc])) {
                exec(S, w, w.ops[w.pc]);
                w.pc++;
                progress = true;
            }
            if (w.pc < w.ops.size()) done = false;
        }
        if (done) break;
        if (!progress) return -2;
    }
    /* outputs: events grouped by worker in execution order */
    std::vector<orc_event> sorted;
    for (auto &w : S.W)
        for (auto &e : S.ev) if (e.worker == w.id) sorted.push_back(e);
    if (n_events) *n_events = (int)sorted.size();
    if (events) {
        if ((int)sorted.size() > events_cap) return -3;
        memcpy(events, sorted.data(), sizeof(orc_event) * sorted.size());
    }
    if (version_map) memcpy(version_map, S.vmap.data(), sizeof(int) * S.vmap.size());
    if (losses) memcpy(losses, S.losses.data(), sizeof(float) * M);
    double mk = 0.0, busy = 0.0;
    for (auto &e : S.ev) {
        if (e.end > mk) mk = e.end;
        busy += e.end - e.start;
    }
    if (max_live)
        for (int s = 0; s < n_stages; s++) {
            int m = 0;
            for (int r = 0; r < S.R[s]; r++) m = m > S.W[S.wbase[s] + r].max_live ? m : S.W[S.wbase[s] + r].max_live;
            max_live[s] = m;
        }
    if (makespan) *makespan = mk;
    if (bubble) *bubble = mk > 0 ? 1.0 - busy / ((double)S.W.size() * mk) : 0.0;
    if (S.math && params)
        for (int s = 0; s < n_stages; s++) {
            Worker &w = S.W[S.wbase[s]];
            memcpy(params + S.poff[S.first[s]], w.versions[w.version].data(), sizeof(float) * S.stage_params(s));
        }
    return 0;
}

/*
 * §3.1 partitioner, single topology level (R10-R16):
 *   A0(i->j) = sum_{l=i..j} T_l (left to right)
 *   T(i->j,m) = max(A0(i->j), C) / m with C = 2 (m-1) sum w_l / B          (comm_model 0, literal)
 *                                        or C = 2 (m-1) sum w_l / (m B)    (comm_model 1)
 *   A(i->j,m) = min( T(i->j,m),  min_{i<=s<j} min_{1<=m'<m} max(A(i->s,m-m'), 2 a_s / B, T(s+1->j,m')) )
 * Ties: single stage first, then s ascending, then m' ascending, strict < (R15).
 * max_replicas (0 = unconstrained) bounds every stage's replication factor.
 * Outputs stage_last[], stage_replicas[] (input stage first), noam = ceil(gpus / R_0).
 * Returns 0, -1 invalid, -7 infeasible.
 */
int orc_plan(const double *T, const unsigned long long *a, const unsigned long long *w, int N, int gpus,
             double bandwidth, int max_replicas, int comm_model, int *n_stages, int *stage_last,
             int *stage_replicas, int *noam, double *slowest) {
    if (N < 1 || gpus < 1) return -1;
    double Bw = bandwidth > 0 ? bandwidth : 900e9;
    int maxr = max_replicas > 0 ? max_replicas : gpus;
    const double INF = 1e300;
    auto idx = [&](int i, int j, int m) { return ((long)i * N + j) * (gpus + 1) + m; };
    std::vector<double> A((long)N * N * (gpus + 1), INF);
    std::vector<int> bs((long)N * N * (gpus + 1), -1), bm((long)N * N * (gpus + 1), -1);
    auto Tst = [&](int i, int j, int m) -> double {
        if (m > maxr) return INF;
        double comp = 0.0;
        for (int l = i; l <= j; l++) comp += T[l];
        double wsum = 0.0;
        for (int l = i; l <= j; l++) wsum += (double)w[l];
        double comm = comm_model == 1 ? 2.0 * (m - 1) * wsum / ((double)m * Bw) : 2.0 * (m - 1) * wsum / Bw;
        double mx = comp > comm ? comp : comm;
        return mx / (double)m;
    };
    for (int len = 1; len <= N; len++)
        for (int i = 0; i + len - 1 < N; i++) {
            int j = i + len - 1;
            for (int m = 1; m <= gpus; m++) {
                double best = Tst(i, j, m);
                int bsv = -1, bmv = -1;
                for (int s = i; s < j; s++)
                    for (int mp = 1; mp < m; mp++) {
                        double x = A[idx(i, s, m - mp)];
                        double c = 2.0 * (double)a[s] / Bw;
                        double y = Tst(s + 1, j, mp);
                        double v = x;
                        if (c > v) v = c;
                        if (y > v) v = y;
                        if (v < best) { best = v; bsv = s; bmv = mp; }
                    }
                A[idx(i, j, m)] = best; bs[idx(i, j, m)] = bsv; bm[idx(i, j, m)] = bmv;
            }
        }
    double best = A[idx(0, N - 1, gpus)];
    if (!(best < INF)) return -7;
    /* backtrack: peel the last stage off repeatedly */
    std::vector<int> lasts, reps;
    int j = N - 1, m = gpus;
    for (;;) {
        int s = bs[idx(0, j, m)], mp = bm[idx(0, j, m)];
        if (s < 0) { lasts.push_back(j); reps.push_back(m); break; }
        lasts.push_back(j); reps.push_back(mp);
        j = s; m = m - mp;
    }
    int n = (int)lasts.size();
    for (int q = 0; q < n; q++) { stage_last[q] = lasts[n - 1 - q]; stage_replicas[q] = reps[n - 1 - q]; }
    *n_stages = n;
    *noam = ceil_div(gpus, stage_replicas[0]);
    *slowest = best;
    return 0;
}

/*
 * §3.1 partitioner over a hierarchical topology (Fig. 7): level k (k = 1..L) is
 * made of m_k components of level k-1 joined by links of bandwidth B_k; level 0 is one GPU
 * (m_0 = 1).  Solved from the lowest level up (L881-885):
 *   A^0(i->j, m_0) = sum_{l=i..j} T_l                                         (L967-971)
 *   T^k(i->j, m) = max( A^{k-1}(i->j, m_{k-1}), C_k ) / m,  C_k = 2 (m-1) sum w_l / B_k
 *                                          (comm_model 1: C_k / m)             (L903-927)
 *   A^k(i->j, m) = min( T^k(i->j, m),
 *                  min_{i<=s<j} min_{1<=m'<m} max( A^k(i->s, m-m'), 2 a_s / B_k, T^k(s+1->j, m') ) )
 *                                                                              (L931-941)
 *   A^k(i->j, 1) = A^{k-1}(i->j, m_{k-1}) follows from T^k(i->j, 1) (L971-975).
 * Ties as in orc_plan.  max_replicas bounds the m chosen at every level.  The plan is
 * returned flattened: a level-k stage replicated m' times over level-(k-1) components runs
 * the level-(k-1) plan of its layers inside each component, so each of those sub-stages
 * becomes one stage replicated m' x (its own replication).  gpus = prod m_k.
 */
int orc_plan_levels(const double *T, const unsigned long long *a, const unsigned long long *w, int N, int n_levels,
                    const int *level_m, const double *level_bw, int max_replicas, int comm_model, int *n_stages,
                    int *stage_last, int *stage_replicas, int *noam, double *slowest) {
    if (N < 1 || n_levels < 1) return -1;
    int gpus = 1;
    for (int k = 0; k < n_levels; k++) {
        if (level_m[k] < 1 || !(level_bw[k] > 0)) return -1;
        gpus *= level_m[k];
    }
    const double INF = 1e300;
    /* per level: A[i][j][m], argmin split and m' */
    struct Level { int mk; double bw; std::vector<double> A; std::vector<int> bs, bm; };
    std::vector<Level> lev(n_levels);
    std::vector<double> below((long)N * N, 0.0);  /* A^{k-1}(i->j, m_{k-1}) */
    for (int i = 0; i < N; i++)
        for (int j = i; j < N; j++) {
            double s = 0.0;
            for (int l = i; l <= j; l++) s += T[l];
            below[(long)i * N + j] = s;
        }
    for (int k = 0; k < n_levels; k++) {
        Level &L = lev[k];
        L.mk = level_m[k];
        L.bw = level_bw[k];
        const int M1 = L.mk + 1;
        L.A.assign((long)N * N * M1, INF);
        L.bs.assign((long)N * N * M1, -1);
        L.bm.assign((long)N * N * M1, -1);
        auto id = [&](int i, int j, int m) { return ((long)i * N + j) * M1 + m; };
        auto Tk = [&](int i, int j, int m) -> double {
            if (max_replicas > 0 && m > max_replicas) return INF;
            double wsum = 0.0;
            for (int l = i; l <= j; l++) wsum += (double)w[l];
            double comm = comm_model == 1 ? 2.0 * (m - 1) * wsum / ((double)m * L.bw) : 2.0 * (m - 1) * wsum / L.bw;
            double comp = below[(long)i * N + j];
            if (!(comp < INF)) return INF;  /* no level-(k-1) plan for these layers: none here either */
            return (comp > comm ? comp : comm) / (double)m;
        };
        for (int len = 1; len <= N; len++)
            for (int i = 0; i + len - 1 < N; i++) {
                int j = i + len - 1;
                for (int m = 1; m <= L.mk; m++) {
                    double best = Tk(i, j, m);
                    int bsv = -1, bmv = -1;
                    for (int s = i; s < j; s++)
                        for (int mp = 1; mp < m; mp++) {
                            double v = L.A[id(i, s, m - mp)];
                            double c = 2.0 * (double)a[s] / L.bw;
                            double y = Tk(s + 1, j, mp);
                            if (c > v) v = c;
                            if (y > v) v = y;
                            if (v < best) { best = v; bsv = s; bmv = mp; }
                        }
                    L.A[id(i, j, m)] = best; L.bs[id(i, j, m)] = bsv; L.bm[id(i, j, m)] = bmv;
                }
            }
        for (int i = 0; i < N; i++)
            for (int j = i; j < N; j++) below[(long)i * N + j] = L.A[id(i, j, L.mk)];
    }
    const Level &top = lev[n_levels - 1];
    double best = top.A[((long)0 * N + (N - 1)) * (top.mk + 1) + top.mk];
    if (!(best < INF)) return -7;
    /* expand level k's plan of layers i..j on m components, each stage replicated `mult` more times */
    std::vector<int> lasts, reps;
    std::function<void(int, int, int, int, int)> expand = [&](int k, int i, int j, int m, int mult) {
        const Level &L = lev[k];
        auto id = [&](int ii, int jj, int mm) { return ((long)ii * N + jj) * (L.mk + 1) + mm; };
        std::vector<int> sl, sr;  /* this level's stages, last first */
        int jj = j, mm = m;
        for (;;) {
            int s = L.bs[id(i, jj, mm)], mp = L.bm[id(i, jj, mm)];
            if (s < 0) { sl.push_back(jj); sr.push_back(mm); break; }
            sl.push_back(jj); sr.push_back(mp);
            jj = s; mm -= mp;
        }
        int first = i;
        for (int q = (int)sl.size() - 1; q >= 0; q--) {
            if (k == 0) { lasts.push_back(sl[q]); reps.push_back(mult * sr[q]); }
            else expand(k - 1, first, sl[q], lev[k - 1].mk, mult * sr[q]);
            first = sl[q] + 1;
        }
    };
    expand(n_levels - 1, 0, N - 1, top.mk, 1);
    int n = (int)lasts.size();
    for (int q = 0; q < n; q++) { stage_last[q] = lasts[q]; stage_replicas[q] = reps[q]; }
    *n_stages = n;
    *noam = ceil_div(gpus, stage_replicas[0]);
    *slowest = best;
    return 0;
}

}  // extern "C"
