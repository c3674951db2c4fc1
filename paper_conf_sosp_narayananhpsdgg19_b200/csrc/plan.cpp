// plan.cpp -- pd_plan: PipeDream's §3.1 partitioner, host side.
//
// By default a single topology level on an NVSwitch node (R13: m_0 = 1, m_1 =
// #GPUs, B_1 = per-GPU NVLink bandwidth); pd_plan_opts.num_levels > 1 gives Fig. 7's
// hierarchy (servers of GPUs, ...), solved level by level from the lowest (L881-885) with
// the level below's whole-component time in place of sum T_l.  Formulas as read in
// DESIGN.md R10-R16 (level k, B = B_k):
//   T(i->j, m) = max( sum_{l=i..j} T_l ,  C(i->j, m) ) / m                       (L903-927)
//     C = 2 (m-1) sum w_l / B            (comm_model 0, literal)
//     C = 2 (m-1) sum w_l / (m B)        (comm_model 1, per-link ring)
//   A(i->j, m) = min( T(i->j, m),
//                     min_{i<=s<j} min_{1<=m'<m} max( A(i->s, m-m'), 2 a_s / B, T(s+1->j, m') ) )
//                                                                                (L931-941)
// Tie order (R15): single stage first, then s ascending, then m' ascending; strict <.
// Sums are accumulated left to right in double.  O(N^3 m^2) (L977-983).
#include <cmath>
#include <cstring>
#include <vector>

#include "pd_internal.h"

namespace pd {

namespace {
// One topology level k: the DP over A^k(i->j, m), m = 1..mk, on top of the level below's
// whole-component times below(i, j) = A^{k-1}(i->j, m_{k-1}) (level 0: sum of T_l).
struct Level {
    int N = 0, mk = 0, maxr = 0, comm = 0;
    double bw = 0;
    const pd_layer_profile *prof = nullptr;
    const std::vector<double> *below = nullptr;  // [i * N + j]
    std::vector<double> best;    // A^k(i->j, m)
    std::vector<int> split, rep; // argmin: split s (-1 => single stage), m'
    size_t at(int i, int j, int m) const { return ((size_t)i * N + j) * (mk + 1) + m; }

    double stage_time(int i, int j, int m) const {
        if (m > maxr) return HUGE_VAL;
        double wbytes = 0.0;
        for (int l = i; l <= j; ++l) wbytes += (double)prof[l].param_bytes;
        const double compute = (*below)[(size_t)i * N + j];
        const double sync = comm == 1 ? 2.0 * (m - 1) * wbytes / ((double)m * bw)
                                      : 2.0 * (m - 1) * wbytes / bw;
        return (compute > sync ? compute : sync) / (double)m;
    }

    void solve() {
        const size_t cells = (size_t)N * N * (mk + 1);
        best.assign(cells, HUGE_VAL);
        split.assign(cells, -1);
        rep.assign(cells, -1);
        for (int len = 1; len <= N; ++len) {
            for (int i = 0; i + len <= N; ++i) {
                const int j = i + len - 1;
                for (int m = 1; m <= mk; ++m) {
                    double v = stage_time(i, j, m);  // the whole range as one (replicated) stage
                    int bs = -1, bm = -1;
                    for (int s = i; s < j; ++s) {
                        const double boundary = 2.0 * (double)prof[s].act_bytes / bw;
                        for (int mp = 1; mp < m; ++mp) {
                            double cand = best[at(i, s, m - mp)];
                            if (boundary > cand) cand = boundary;
                            const double last = stage_time(s + 1, j, mp);
                            if (last > cand) cand = last;
                            if (cand < v) {
                                v = cand;
                                bs = s;
                                bm = mp;
                            }
                        }
                    }
                    best[at(i, j, m)] = v;
                    split[at(i, j, m)] = bs;
                    rep[at(i, j, m)] = bm;
                }
            }
        }
    }
};

// Appends the flat stages of level k's plan for layers i..j on m components, every stage's
// replication multiplied by `mult` (the replication of the enclosing higher-level stages).
void flatten(const std::vector<Level> &lev, int k, int i, int j, int m, int mult, std::vector<int> &last_layer,
             std::vector<int> &reps) {
    const Level &L = lev[k];
    std::vector<int> sl, sr;  // this level's stages, output stage first
    int jj = j, mm = m;
    while (true) {
        const int s = L.split[L.at(i, jj, mm)];
        if (s < 0) {
            sl.push_back(jj);
            sr.push_back(mm);
            break;
        }
        const int mp = L.rep[L.at(i, jj, mm)];
        sl.push_back(jj);
        sr.push_back(mp);
        jj = s;
        mm -= mp;
    }
    int first = i;
    for (int q = (int)sl.size() - 1; q >= 0; --q) {
        if (k == 0) {
            last_layer.push_back(sl[q]);
            reps.push_back(mult * sr[q]);
        } else {
            flatten(lev, k - 1, first, sl[q], lev[k - 1].mk, mult * sr[q], last_layer, reps);
        }
        first = sl[q] + 1;
    }
}
}  // namespace

pd_status plan_partition(const pd_layer_profile *layers, int N, int G, const pd_plan_opts *opts, pd_plan_t *out) {
    if (!layers || !out || N < 1 || N > 4096 || G < 1 || G > 4096) return PD_EINVAL;
    const int comm = opts ? opts->comm_model : 0;
    if (comm != 0 && comm != 1) return PD_EINVAL;
    const int maxr_opt = (opts && opts->max_replicas > 0) ? opts->max_replicas : 0;
    // the levels, lowest first (one level by default: the NVSwitch node, R13)
    std::vector<int> sizes;
    std::vector<double> bws;
    const int nl = opts ? opts->num_levels : 0;
    if (nl < 0 || nl > PD_MAX_LEVELS) return PD_EINVAL;
    if (nl <= 1) {
        sizes.push_back(G);
        bws.push_back(nl == 1 && opts->level_bw[0] > 0 ? opts->level_bw[0]
                      : (opts && opts->bandwidth_Bps > 0) ? opts->bandwidth_Bps : 900e9);
        if (nl == 1 && opts->level_size[0] != G) return PD_EINVAL;
    } else {
        long prod = 1;
        for (int k = 0; k < nl; ++k) {
            if (opts->level_size[k] < 1 || !(opts->level_bw[k] > 0)) return PD_EINVAL;
            sizes.push_back(opts->level_size[k]);
            bws.push_back(opts->level_bw[k]);
            prod *= opts->level_size[k];
        }
        if (prod != G) return PD_EINVAL;
    }
    std::vector<Level> lev(sizes.size());
    std::vector<double> below((size_t)N * N, 0.0);
    for (int i = 0; i < N; ++i) {
        double acc = 0.0;  // A^0(i->j) = sum of T_l, left to right (R16)
        for (int j = i; j < N; ++j) {
            acc += layers[j].compute_s;
            below[(size_t)i * N + j] = acc;
        }
    }
    for (size_t k = 0; k < lev.size(); ++k) {
        Level &L = lev[k];
        L.N = N;
        L.mk = sizes[k];
        L.bw = bws[k];
        L.maxr = maxr_opt > 0 ? maxr_opt : L.mk;
        L.comm = comm;
        L.prof = layers;
        L.below = &below;
        L.solve();
        std::vector<double> next((size_t)N * N);
        for (int i = 0; i < N; ++i)
            for (int j = i; j < N; ++j) next[(size_t)i * N + j] = L.best[L.at(i, j, L.mk)];
        below.swap(next);
        L.below = nullptr;
    }
    const Level &top = lev.back();
    const double total = top.best[top.at(0, N - 1, top.mk)];
    if (!std::isfinite(total)) return PD_EINFEASIBLE;

    std::vector<int> last_layer, reps;
    flatten(lev, (int)lev.size() - 1, 0, N - 1, top.mk, 1, last_layer, reps);
    const int n = (int)last_layer.size();
    if (n > PD_MAX_STAGES) return PD_EUNSUPPORTED;
    pd_plan_t p;
    std::memset(&p, 0, sizeof(p));
    p.num_stages = n;
    int gpu = 0, first = 0;
    for (int q = 0; q < n; ++q) {
        pd_stage_desc &sd = p.stage[q];
        sd.first_layer = first;
        sd.last_layer = last_layer[q];
        sd.replicas = reps[q];
        sd.first_gpu = gpu;  // consecutive GPU ids in stage order (R18)
        gpu += sd.replicas;
        first = sd.last_layer + 1;
    }
    p.noam = (G + p.stage[0].replicas - 1) / p.stage[0].replicas;  // ceil (L1021, R1)
    p.slowest_stage_s = total;
    *out = p;
    return PD_OK;
}

}  // namespace pd

extern "C" pd_status pd_plan(const pd_layer_profile *layers, int num_layers, int num_gpus, const pd_plan_opts *opts,
                             pd_plan_t *out) {
    return pd::plan_partition(layers, num_layers, num_gpus, opts, out);
}
