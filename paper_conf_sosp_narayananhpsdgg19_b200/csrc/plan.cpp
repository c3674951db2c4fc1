// plan.cpp -- pd_plan: PipeDream's §3.1 partitioner, host side.
//
// Single topology level on an NVSwitch node (R13: m_0 = 1, m_1 = #GPUs, B_1 =
// per-GPU NVLink bandwidth; the hierarchical levels of Fig. 7 collapse because every GPU
// pair has the same bandwidth).  Formulas as read in DESIGN.md R10-R16:
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
struct Dp {
    int N, G, maxr, comm;
    double bw;
    const pd_layer_profile *prof;
    std::vector<double> best;   // A(i->j, m)
    std::vector<int> split, rep; // argmin: split s (-1 => single stage), m'
    size_t at(int i, int j, int m) const { return ((size_t)i * N + j) * (G + 1) + m; }

    double stage_time(int i, int j, int m) const {
        if (m > maxr) return HUGE_VAL;
        double compute = 0.0, wbytes = 0.0;
        for (int l = i; l <= j; ++l) compute += prof[l].compute_s;
        for (int l = i; l <= j; ++l) wbytes += (double)prof[l].param_bytes;
        const double sync = comm == 1 ? 2.0 * (m - 1) * wbytes / ((double)m * bw)
                                      : 2.0 * (m - 1) * wbytes / bw;
        return (compute > sync ? compute : sync) / (double)m;
    }
};
}  // namespace

pd_status plan_partition(const pd_layer_profile *layers, int N, int G, const pd_plan_opts *opts, pd_plan_t *out) {
    if (!layers || !out || N < 1 || N > 4096 || G < 1 || G > 4096) return PD_EINVAL;
    Dp d;
    d.N = N;
    d.G = G;
    d.prof = layers;
    d.bw = (opts && opts->bandwidth_Bps > 0) ? opts->bandwidth_Bps : 900e9;
    d.maxr = (opts && opts->max_replicas > 0) ? opts->max_replicas : G;
    d.comm = opts ? opts->comm_model : 0;
    if (d.comm != 0 && d.comm != 1) return PD_EINVAL;
    const size_t cells = (size_t)N * N * (G + 1);
    d.best.assign(cells, HUGE_VAL);
    d.split.assign(cells, -1);
    d.rep.assign(cells, -1);

    for (int len = 1; len <= N; ++len) {
        for (int i = 0; i + len <= N; ++i) {
            const int j = i + len - 1;
            for (int m = 1; m <= G; ++m) {
                double v = d.stage_time(i, j, m);  // the whole range as one (replicated) stage
                int bs = -1, bm = -1;
                for (int s = i; s < j; ++s) {
                    const double boundary = 2.0 * (double)layers[s].act_bytes / d.bw;
                    for (int mp = 1; mp < m; ++mp) {
                        double cand = d.best[d.at(i, s, m - mp)];
                        if (boundary > cand) cand = boundary;
                        const double last = d.stage_time(s + 1, j, mp);
                        if (last > cand) cand = last;
                        if (cand < v) {
                            v = cand;
                            bs = s;
                            bm = mp;
                        }
                    }
                }
                d.best[d.at(i, j, m)] = v;
                d.split[d.at(i, j, m)] = bs;
                d.rep[d.at(i, j, m)] = bm;
            }
        }
    }
    const double total = d.best[d.at(0, N - 1, G)];
    if (!std::isfinite(total)) return PD_EINFEASIBLE;

    // Walk the argmin chain from the output stage back to the input stage.
    std::vector<int> last_layer, reps;
    int j = N - 1, m = G;
    while (true) {
        const int s = d.split[d.at(0, j, m)];
        if (s < 0) {
            last_layer.push_back(j);
            reps.push_back(m);
            break;
        }
        const int mp = d.rep[d.at(0, j, m)];
        last_layer.push_back(j);
        reps.push_back(mp);
        j = s;
        m -= mp;
    }
    const int n = (int)last_layer.size();
    if (n > PD_MAX_STAGES) return PD_EUNSUPPORTED;
    pd_plan_t p;
    std::memset(&p, 0, sizeof(p));
    p.num_stages = n;
    int gpu = 0, first = 0;
    for (int q = 0; q < n; ++q) {
        pd_stage_desc &sd = p.stage[q];
        sd.first_layer = first;
        sd.last_layer = last_layer[n - 1 - q];
        sd.replicas = reps[n - 1 - q];
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
