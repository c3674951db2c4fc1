"""PipeDream's profile -> optimize -> run loop on B200.

    python tools/plan_sweep.py [--config mlp4096|gnmt8|gnmt16|vgg16] [--gpus 1 2 4 8]
                               [--depth-sweep] [--json out.json]

1. Profiler (L841-847): pd_profile measures (T_l, a_l, w_l) of every layer on this GPU.
2. Optimizer (L855-985): pd_plan on that profile for each GPU count -- unconstrained and
   straight (max_replicas = 1) -- with the predicted throughput B / A(0 -> N, m).
3. Predicted vs real (Fig. 15) where this host can run the plan: the 1-GPU
   plan is run at full speed and its samples/s set against the prediction.
3b. Predicted vs real beyond one GPU with --real-stages: every stage of each straight plan is
   run alone on this GPU (pd_stage_solo: neighbours replaced by infinitely fast stand-ins),
   and B * min_s R_s / t_s of the measured stage times is set against the optimizer's
   B / A(0 -> N, m) (the pipeline's throughput is its slowest stage's, L775-777; transfers
   and the fill/drain bubble are not in either number).
4. Depth sweep (Fig. 18) with --depth-sweep: a straight pipeline of the
   largest --gpus count run as virtual workers on this GPU with pd_run(M, D) for
   D = 1 .. n+2 -- per-stage stash memory (weight versions k_s(D) and activation rings, from
   the runtime's own allocation rule) and the measured bubble.  Throughput of virtual
   workers sharing one GPU is NOT a multi-GPU number and is labelled so.
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402
import paper_conf_sosp_narayananhpsdgg19_b200 as pd  # noqa: E402
from paper_conf_sosp_narayananhpsdgg19_b200.session import Pipeline  # noqa: E402


def layer_in_bytes(L, B):
    if L.kind in (synth.CONV3X3, synth.MAXPOOL2):
        return B * L.height * L.width * L.in_ * 2
    if L.kind == synth.EMBEDDING:
        return B * L.seq_len * 4
    return B * (L.seq_len or 1) * L.in_ * 2


def stage_memory(layers, plan, B, k, optimizer):
    """Per-stage device bytes that depend on the pipeline depth (bf16 path): k_s weight
    versions (bf16), fp32 master (+ Adam m, v), k_s-deep stash of every inner layer's input,
    a receive ring of k_s + 1 input slots (straight plans)."""
    out = []
    for s, (first, last, _r, _g) in enumerate(plan.stages):
        P = sum(synth.param_count(layers[l]) for l in range(first, last + 1))
        w = k[s] * P * 2 + P * 4 * (3 if optimizer == synth.ADAM else 1)
        act = k[s] * sum(layer_in_bytes(layers[l], B) for l in range(first + 1, last + 1))
        recv = (k[s] + 1) * layer_in_bytes(layers[first], B) if s > 0 else 0
        out.append({"stage": s, "k": k[s], "weights_gb": w / 1e9, "activations_gb": (act + recv) / 1e9})
    return out


def run_real(wl, plan, M, noam=0, max_depth=0, repeats=3):
    p0 = synth.init_params(wl.layers)
    data = synth.make_data(wl, 8)
    with Pipeline(plan, wl.layers, p0, dtype=pd.PD_BF16, optimizer=wl.optimizer, lr=wl.lr, minibatch=wl.batch,
                  record_trace=2, max_depth=max_depth) as P:
        P.set_data(*data, 8)
        P.set_timing(2, 0)
        P.run(M, noam)  # warm-up
        ms, bub = [], []
        for _ in range(repeats):
            P.run(M, noam)
            st = P.stats()
            ms.append(st["run_ms"])
            bub.append(st["bubble"])
    return M * wl.batch / (float(np.median(ms)) / 1e3), float(np.mean(bub))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="mlp4096")
    ap.add_argument("--gpus", type=int, nargs="+", default=[1, 2, 4, 8])
    ap.add_argument("--profile-minibatches", type=int, default=8)
    ap.add_argument("--depth-sweep", action="store_true")
    ap.add_argument("--real-stages", action="store_true")
    ap.add_argument("--json", default="")
    a = ap.parse_args()
    wl = synth.workload(a.config)
    L, B = wl.layers, wl.batch
    res = {"config": a.config, "minibatch": B}

    t0 = time.perf_counter()
    T, act, w = pd.pd_profile(L, pd.PD_BF16, wl.optimizer, wl.lr, B, 0, a.profile_minibatches)
    res["profile"] = {"T_s": T, "a_bytes": act, "w_bytes": w, "seconds": time.perf_counter() - t0}
    print(f"profile ({time.perf_counter() - t0:.1f} s): sum T_l = {sum(T) * 1e3:.3f} ms per minibatch")
    for l, Ly in enumerate(L):
        print(f"  layer {l:2d} kind {Ly.kind} T {T[l] * 1e6:9.1f} us  a {act[l] / 1e6:8.2f} MB  w {w[l] / 1e6:8.2f} MB")

    plans = []
    for N in a.gpus:
        for mr, tag in ((0, "free"), (1, "straight")):
            try:
                t1 = time.perf_counter()
                p = pd.pd_plan(T, act, w, N, max_replicas=mr)
                dt = time.perf_counter() - t1
            except pd.PDError as e:
                print(f"N={N} {tag}: {e}")
                continue
            pred = B / p.slowest_stage_s
            desc = "-".join(str(s[2]) for s in p.stages) + " " + str([s[1] - s[0] + 1 for s in p.stages])
            print(f"N={N} {tag:8s} plan {desc:30s} NOAM {p.noam}  predicted {pred:10.1f} samples/s "
                  f"(optimizer {dt * 1e3:.1f} ms)")
            plans.append({"gpus": N, "kind": tag, "stages": p.stages, "noam": p.noam,
                          "predicted_samples_per_s": pred, "optimizer_ms": dt * 1e3})
    res["plans"] = plans

    # predicted vs real where this host can run the plan (1 GPU)
    one = pd.Plan.manual([len(L) - 1], [1])
    real, _ = run_real(wl, one, 8)
    pred = B / sum(T)
    print(f"1 GPU: predicted {pred:.1f} samples/s (sum of serialised per-layer times), real {real:.1f} "
          f"(ratio {real / pred:.2f}; the real run overlaps dW with dX and replays graphs)")
    res["predicted_vs_real_1gpu"] = {"predicted": pred, "real": real, "ratio": real / pred}

    if a.real_stages:
        import bench
        p0 = synth.init_params(L)
        data = synth.make_data(wl, 8)
        for pl in plans:
            if pl["kind"] != "straight" or pl["gpus"] < 2:
                continue
            p = pd.Plan(pl["stages"], pl["noam"], 0.0)
            ts = []
            for s_ in range(len(p.stages)):
                r = bench.solo_stage(p, s_, L, wl, p0, data, 8, 8 * p.stages[s_][2], runs=2, warm=1, profile=False)
                ts.append(r["ms_per_minibatch"])
            real = B * min(st[2] / (t / 1e3) for st, t in zip(p.stages, ts))
            pl["stage_ms_solo"] = ts
            pl["real_from_stages_samples_per_s"] = real
            pl["real_over_predicted"] = real / pl["predicted_samples_per_s"]
            print(f"N={pl['gpus']} straight: stage ms {[round(t, 3) for t in ts]} -> {real:10.1f} samples/s "
                  f"(predicted {pl['predicted_samples_per_s']:10.1f}, ratio {real / pl['predicted_samples_per_s']:.2f})")

    if a.depth_sweep:
        N = max(a.gpus)
        p = pd.pd_plan(T, act, w, N, max_replicas=1)
        n = len(p.stages)
        sweep = []
        for D in range(1, n + 3):
            k = pd.pd_inflight(p, D)
            M = 4 * n
            sps, bub = run_real(wl, p, M, noam=D, max_depth=n + 2, repeats=2)
            mem = stage_memory(L, p, B, k, wl.optimizer)
            print(f"depth {D}: k {k}  bubble {100 * bub:5.1f} %  virtual-worker samples/s {sps:9.1f}  "
                  f"stage-0 stash {mem[0]['weights_gb']:.2f} GB weights + {mem[0]['activations_gb']:.3f} GB act")
            sweep.append({"depth": D, "k": k, "bubble": bub, "virtual_workers_samples_per_s": sps, "memory": mem})
        res["depth_sweep"] = {"gpus": N, "plan": p.stages, "noam": p.noam, "points": sweep,
                              "note": "all stages as virtual workers on ONE GPU: bubble and memory are the "
                                      "pipeline's, samples/s is not a multi-GPU number"}
    if a.json:
        json.dump(res, open(a.json, "w"), indent=1)


if __name__ == "__main__":
    main()
