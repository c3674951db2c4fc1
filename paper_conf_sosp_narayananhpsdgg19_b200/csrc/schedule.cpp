// schedule.cpp -- the static 1F1B-RR op lists (§3.2).
//
// Worker (s, r) owns the minibatches t = r, r + R_s, r + 2 R_s, ... (deterministic
// round-robin by minibatch id, L1067-1077, R4).  With k = min(k_s, M_r) its list is
//     F(t_0) ... F(t_{k-1})                          startup: admit k_s minibatches
//     B(t_j) U F(t_{j+k})    for j = 0 .. M_r-k-1    steady state: one backward, one forward
//     B(t_j) U               for the remaining j     drain
// where U (the weight update of the backward just run) precedes the next forward so the
// forward sees the latest version (L237-241).  k_s = ceil(W_{>=s} / R_s), NOAM = k_0
// (L1021, ceiling per R1; stages s > 0 per R2); a depth override D (straight plans only)
// gives k_s = max(1, D - s) and k_{n-1} = 1 (R19).
#include "pd_internal.h"

namespace pd {

pd_status inflight_counts(const pd_plan_t &plan, int depth, std::vector<int> &k) {
    const int n = plan.num_stages;
    bool straight = true;
    for (int s = 0; s < n; ++s) straight = straight && plan.stage[s].replicas == 1;
    if (depth < 0 || (depth > 0 && !straight)) return PD_EINVAL;
    k.assign(n, 1);
    for (int s = 0; s < n; ++s) {
        if (depth > 0) {
            k[s] = (s == n - 1) ? 1 : (depth - s > 1 ? depth - s : 1);
        } else {
            int downstream = 0;  // W_{>=s}
            for (int q = s; q < n; ++q) downstream += plan.stage[q].replicas;
            k[s] = (downstream + plan.stage[s].replicas - 1) / plan.stage[s].replicas;
        }
    }
    return PD_OK;
}

std::vector<Op> worker_ops(int R_s, int replica, int k_s, int M) {
    std::vector<int> mine;
    for (int t = replica; t < M; t += R_s) mine.push_back(t);
    const int Mr = (int)mine.size();
    const int k = k_s < Mr ? k_s : Mr;
    std::vector<Op> ops;
    ops.reserve(3 * Mr);
    for (int j = 0; j < k; ++j) ops.push_back({'F', mine[j], j});
    for (int j = 0; j < Mr; ++j) {
        ops.push_back({'B', mine[j], j});
        ops.push_back({'U', mine[j], j});
        if (j + k < Mr) ops.push_back({'F', mine[j + k], j + k});
    }
    return ops;
}

// GPipe comparison schedule (§5.4; R27), straight plans: flush groups of
// D minibatches.  Stages s < n-1: F(t) for the group, then B(t) for the group in t order; the
// last stage: F(t) B(t) back to back (its backward starts immediately, L719-721); one U per
// group (Op.j = group index, Op.t = the group's last minibatch) applies the aggregated
// gradient (L1277-1279).  F / B carry j = t (one replica).
std::vector<Op> gpipe_ops(bool last_stage, int D, int M) {
    std::vector<Op> ops;
    ops.reserve(2 * M + M / D + 1);
    for (int g = 0; g * D < M; ++g) {
        const int t0 = g * D, t1 = t0 + D;
        if (last_stage) {
            for (int t = t0; t < t1; ++t) {
                ops.push_back({'F', t, t});
                ops.push_back({'B', t, t});
            }
        } else {
            for (int t = t0; t < t1; ++t) ops.push_back({'F', t, t});
            for (int t = t0; t < t1; ++t) ops.push_back({'B', t, t});
        }
        ops.push_back({'U', t1 - 1, g});
    }
    return ops;
}

int recv_ring_depth(const pd_plan_t &plan, const std::vector<int> &k, int s) {
    // An activation for t lives in stage s's ring from F(s-1, t) until B(s, t).  The
    // producer replica runs F(t_{j+k}) only after B(t_j), which waits for B(s, t_j), so at
    // most k_{s-1} R_{s-1} minibatches are live across the producers, spread round-robin
    // over R_s consumers.
    const int Rp = plan.stage[s - 1].replicas, Rc = plan.stage[s].replicas;
    return (k[s - 1] * Rp + Rc - 1) / Rc;
}

}  // namespace pd
