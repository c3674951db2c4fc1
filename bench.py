#!/usr/bin/env python
"""Benchmark of the B200-native PipeDream hot path (1F1B + weight stashing).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config mlp4096] [--impl reference]

One step = one pd_run over `--minibatches` minibatches of the BASELINE.json configs[1]
workload (16 x Linear(4096)+ReLU -> CE(4096), minibatch 256, bf16, SGD): startup, steady
state and drain of the 1F1B pipeline, with inputs already resident in HBM (a ring of 8
synthetic minibatches).  N = 1 is a single stage (plain SGD, k = 1, P1); N > 1 is
the straight pipeline pd_plan(max_replicas = 1) returns for N GPUs, one process per GPU
(torchrun), activations/gradients over NVLink peer stores (CUDA IPC).

Prints ONE JSON line (rank 0).  `value` = samples/s of the whole job, device time of each
step = max over ranks of the library's per-run CUDA-event span.  `e2e` repeats the
measurement through the public API with host inputs (pinned) copied in and the losses read
back inside every step.  `roofline` reports the dominant kernel (the dW GEMM with the fused
SGD update -- HBM-bound) against MEASURED_PEAKS.json.  `cpu_baseline` times the oracle.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")

import numpy as np  # noqa: E402

METRIC = "samples/sec at 1/2/4/8 B200 (1F1B+stash); bubble %; per-stage tensor-pipe util"
WORKLOAD_DESC = {
    "mlp4096": "mlp4096: BASELINE configs[1] 16 x Linear(4096)+ReLU -> CE(4096)",
    "gnmt8": "gnmt8: BASELINE configs[2] Emb(32000,1024) -> 8 x LSTM(1024), T=50 -> Linear(1024,32000) -> CE",
    "gnmt16": "gnmt16: BASELINE configs[4] Emb(32000,1024) -> 16 x LSTM(1024), T=50 -> Linear(1024,32000) -> CE",
    "vgg16": "vgg16: BASELINE configs[3] VGG-16 224x224 NHWC, 13 conv3x3 + 5 maxpool + FC 4096/4096/1000",
}


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return {"hbm_gbs": d["hbm_gbs"], "bf16_tflops": d["bf16_tflops"],
                "bf16_tflops_sustained": d.get("bf16_tflops_sustained", d["bf16_tflops"]), "source": "measured"}
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0, "source": "fallback"}


class Clocks:
    """Samples nvidia-smi during the timed region (clocks line of B200_PROFILING.md)."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index, self.rows, self.proc = index, [], None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except FileNotFoundError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)  # at least one sample after the timed region
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.t.join(timeout=2)
        sm = [float(r[1]) for r in self.rows if len(r) > 2 and r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if len(r) > 2 and r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            for nm, v in zip(names, r[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(self.rows)}


# ----------------------------------------------------------------------------- workload

def layer_flops(L, B):
    """Algorithmic fwd+bwd FLOPs of one layer for one minibatch (2 fwd + 4 bwd per MAC)."""
    import synth
    if L.kind == synth.LINEAR:
        return 6.0 * B * (L.seq_len or 1) * L.in_ * L.out
    if L.kind == synth.LSTM:
        return 6.0 * B * L.seq_len * 4 * L.out * (L.in_ + L.out)
    if L.kind == synth.CONV3X3:
        return 6.0 * B * L.height * L.width * L.out * L.in_ * 9
    return 0.0


def layer_out_bytes(L, B):
    import synth
    if L.kind == synth.MAXPOOL2:
        return B * (L.height // 2) * (L.width // 2) * L.in_ * 2
    if L.kind == synth.CONV3X3:
        return B * L.height * L.width * L.out * 2
    return B * (L.seq_len or 1) * L.out * 2


def model_profile(layers, B, peaks):
    """FLOP/byte-proportional per-layer profile for pd_plan (T_l, a_l, w_l, L841-843): compute
    at 60 % of the bf16 peak or the update's HBM bytes, whichever is larger."""
    import synth
    T, a, w = [], [], []
    for L in layers:
        P = synth.param_count(L)
        flop_t = layer_flops(L, B) / (peaks["bf16_tflops"] * 1e12 * 0.6)
        byte_t = 14.0 * P / (peaks["hbm_gbs"] * 1e9)
        T.append(max(flop_t, byte_t, 1e-7))
        a.append(layer_out_bytes(L, B))
        w.append(P * 2)
    return T, a, w


def ncu_traffic(key, config):
    """dram__bytes_read.sum + dram__bytes_write.sum per launch (bytes) of kernel `key` from the
    committed `ncu --set full` capture (profiles/ncu_traffic_r*.json, tools/ncu_traffic.py) of
    this config's launch, or None (a capture of another config's launch does not apply)."""
    import glob
    for path in sorted(glob.glob(os.path.join(ROOT, "profiles", "ncu_traffic_r*.json")), reverse=True):
        d = json.load(open(path))
        if key in d and d[key].get("config", config) == config:
            return d[key]["traffic_MB"] * 1e6
    return None


def choose_plan(config, plan_mode, N, layers, B, peaks):
    """The plan every rank computes independently (deterministic, no exchange): one stage x N
    replicas for N = 1 or --plan dp; VGG-16 as (N-1)-1; otherwise pd_plan(max_replicas=1)."""
    import synth
    import paper_conf_sosp_narayananhpsdgg19_b200 as pd
    if N == 1 or plan_mode == "dp":
        return pd.Plan.manual([len(layers) - 1], [N])
    if config == "vgg16":
        # VGG-16 as (N-1)-1 -- conv stage replicated, FC stage alone
        conv_last = max(i for i, L in enumerate(layers) if L.kind == synth.MAXPOOL2)
        return pd.Plan.manual([conv_last, len(layers) - 1], [N - 1, 1])
    T, a, w = model_profile(layers, B, peaks)
    return pd.pd_plan(T, a, w, N, max_replicas=1)


def dw_update_bytes(L, B):
    """Algorithmic HBM bytes of one dW GEMM with the fused SGD update:
    read G [B][out] and X [B][in] (bf16), read+write the fp32 master, write the bf16 version."""
    return B * L.out * 2 + B * L.in_ * 2 + L.out * L.in_ * (4 + 4 + 2)


def l2_note(layers, optimizer):
    """The timing rule's L2 statement, computed from the workload: bytes every minibatch streams
    (bf16 weights, fp32 master, Adam m and v) against the 126 MB L2."""
    import synth
    P = sum(synth.param_count(L) for L in layers)
    opt = f" + {8 * P / 1e9:.2f} GB Adam m, v" if optimizer == synth.ADAM else ""
    return (f"working set > L2: every minibatch streams {2 * P / 1e9:.2f} GB bf16 weights + "
            f"{4 * P / 1e9:.2f} GB fp32 master{opt} over {len(layers)} layers (126 MB L2), no flush needed")


def stage_roofline(layers, plan, B, peaks, optimizer, nvlink_gbs=900.0):
    """north_star / SURVEY §8(d) per-stage roofline:
        samples/s = B * min_s R_s / max(F_s / P_tensor, H_s / BW_HBM, N_s / BW_NVL)
    F_s = GEMM FLOPs per minibatch (6 per MAC; the model's first layer has no dX);
    H_s = algorithmic HBM bytes per minibatch: bf16 weight reads fwd + bwd (4 B/param),
          the update (fp32 master r+w 8 B + new bf16 version 2 B; Adam m, v r+w +16 B),
          activation stash write + read of every layer input, logits write + read for CE;
    N_s = NVLink bytes: activation out + gradient out (+ ring allreduce 2(R-1)/R grad bytes).
    Peaks: sustained bf16 tensor (a step is a long run) and the measured HBM copy bandwidth."""
    import synth
    per = []
    for s, (first, last, R, _g) in enumerate(plan.stages):
        F = H = Nb = 0.0
        P = 0
        for l in range(first, last + 1):
            L = layers[l]
            f = layer_flops(L, B)
            if l == 0:
                f *= 2.0 / 3.0
            F += f
            p = synth.param_count(L)
            P += p
            H += p * (4 + 10 + (16 if optimizer == synth.ADAM else 0))
            in_bytes = layer_out_bytes(layers[l - 1], B) if l > 0 else 0
            H += 2 * in_bytes
        if last == len(layers) - 1:
            H += 2 * layer_out_bytes(layers[-1], B)
        if last < len(layers) - 1:
            Nb += layer_out_bytes(layers[last], B)
        if first > 0:
            Nb += layer_out_bytes(layers[first - 1], B)
        if R > 1:
            Nb += 2.0 * (R - 1) / R * 4 * P
        t = max(F / (peaks["bf16_tflops_sustained"] * 1e12), H / (peaks["hbm_gbs"] * 1e9), Nb / (nvlink_gbs * 1e9))
        bound = ["tensor", "hbm", "nvlink"][int(np.argmax([F / (peaks["bf16_tflops_sustained"] * 1e12),
                                                            H / (peaks["hbm_gbs"] * 1e9), Nb / (nvlink_gbs * 1e9)]))]
        per.append({"stage": s, "gflop": F / 1e9, "hbm_gb": H / 1e9, "nvlink_mb": Nb / 1e6, "bound": bound,
                    "samples_per_s": B * R / t})
    slow = min(range(len(per)), key=lambda i: per[i]["samples_per_s"])
    return per[slow]["samples_per_s"], slow, per


def class_flops(layers, first, last, B):
    """Algorithmic FLOPs per minibatch of one stage [first, last] split by the runtime's kernel
    classes (pd.KERNEL_CLASSES): 0 forward GEMMs, 1 dX GEMMs, 2 dW GEMMs, 4 / 5 the LSTM
    wavefront kernels (runs of >= 2 equal LSTMs: forward with the input projection folded in,
    backward dh over W_hh plus the inner layers' input gradients), 2 per MAC."""
    import synth
    fl = [0.0] * 8
    l = first
    while l <= last:
        L = layers[l]
        run = 1
        if L.kind == synth.LSTM:
            while (l + run <= last and layers[l + run].kind == synth.LSTM and run < 16 and
                   layers[l + run].in_ == L.out == layers[l + run].out and L.in_ == L.out):
                run += 1
        need_dx = l > 0
        if L.kind == synth.LSTM and run >= 2:
            H, T = L.out, L.seq_len
            fl[4] += run * 2.0 * B * T * 4 * H * 2 * H
            fl[5] += run * 2.0 * B * T * 4 * H * H + (run - 1) * 2.0 * B * T * 4 * H * H
            if need_dx:
                fl[1] += 2.0 * B * T * 4 * H * H
            fl[2] += run * (2.0 * B * T * 4 * H * H + 2.0 * B * (T - 1) * 4 * H * H)
            l += run
            continue
        f = layer_flops(L, B) / 3.0
        fl[0] += f
        fl[2] += f
        if need_dx:
            fl[1] += f
        l += 1
    return fl


def gemm_flops(L, B):
    return 2.0 * B * L.in_ * L.out


def pass_flops(L, B):
    """FLOPs of ONE GEMM pass (forward, dX or dW: 2 per MAC) of layer L for one minibatch."""
    return layer_flops(L, B) / 3.0


# ----------------------------------------------------------------------------- reference arm

def oracle_sample(config, wl, mlp_batch):
    """A bounded sample of the workload for the single-threaded oracle (~0.4-1 GFLOP/s):
    (layers, B, scale, text).  Samples/s of the full workload = scale * B / seconds, where
    `scale` converts the sample's work to whole samples:
      mlp4096   B = mlp_batch samples of the full model (scale 1);
      gnmt*     1 sequence, 2 of its T = 50 tokens (LSTM / classifier work per token is
                constant; scale 2/50);
      vgg16     1 image cropped to 32 x 32 (conv work per pixel is constant; the FC stack is
                < 1 % of VGG-16's FLOPs; scale (32/224)^2)."""
    import synth
    if config in ("gnmt8", "gnmt16"):
        n = sum(1 for L in wl.layers if L.kind == synth.LSTM)
        T = wl.layers[0].seq_len
        return (synth.gnmt(n, 1024, 32000, 2, 1), 1, 2.0 / T,
                f"1 sequence (B=1) of 2 of its {T} tokens through all {len(wl.layers)} layers, scaled by 2/{T}")
    if config == "vgg16":
        return (synth.vgg(synth.VGG16_BLOCKS, 32, 3, [4096, 4096], 1000), 1, (32.0 / 224.0) ** 2,
                "1 image cropped to 32x32 through VGG-16 (FC6 input 1x1x512), scaled by (32/224)^2")
    return wl.layers, mlp_batch, 1.0, f"1 minibatch of B={mlp_batch} (not {wl.batch}) of the full model"


def run_reference(args):
    """--impl reference: the oracle (this tier's reference arm) on the host cores, on a
    bounded sample of the same workload (oracle_sample, a few seconds per step); one JSON line."""
    import oracle
    import synth
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    wl = synth.workload(args.config)
    layers, Bs, scale, text = oracle_sample(args.config, wl, max(1, args.cpu_batch // 8))
    p0 = synth.init_params(layers)
    wl_s = synth.Workload(wl.name, layers, Bs, wl.optimizer, wl.lr)
    data = synth.make_data(wl_s, 1)
    oracle.lib()
    times = []
    with pinned_to_core0() as core:
        for i in range(args.warmup + max(1, args.steps)):
            t0 = time.perf_counter()
            oracle.run(layers, [len(layers) - 1], [1], Bs, 1, p0, data, wl.optimizer, wl.lr)
            if i >= args.warmup:
                times.append(time.perf_counter() - t0)
    per = float(np.median(times))
    value = scale * Bs / per
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "samples/s", "n_gpus": args.gpus,
            "steps": len(times), "warmup": args.warmup, "ms_per_step": per * 1e3, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": WORKLOAD_DESC.get(args.config, args.config) + " run by the CPU oracle (1 stage); "
                                   f"bounded sample per step: {text}", "global_batch": Bs},
            "cpu_baseline": {"value": value, "unit": "samples/s", "cores": 1, "kind": "oracle",
                             "cpu_model": cpu_model(), "nproc": os.cpu_count(), "pinned_core": core,
                             "sample": f"{text}; fwd+bwd+{'Adam' if wl.optimizer else 'SGD'}, single-threaded fp32 "
                                       f"naive loops pinned to core {core}"},
            "e2e": {"value": value, "unit": "samples/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


class pinned_to_core0:
    """taskset -c 0 for the oracle timing (BASELINE.md CPU-baseline plan), restored after."""

    def __enter__(self):
        self.old = os.sched_getaffinity(0)
        os.sched_setaffinity(0, {min(self.old)})
        return min(self.old)

    def __exit__(self, *a):
        os.sched_setaffinity(0, self.old)


def cpu_baseline(args, layers, wl):
    import oracle
    import synth
    layers, Bs, scale, text = oracle_sample(args.config, wl, args.cpu_batch)
    p0 = synth.init_params(layers)
    wl_s = synth.Workload(wl.name, layers, Bs, wl.optimizer, wl.lr)
    data = synth.make_data(wl_s, 1)
    oracle.lib()  # load (and if needed build) outside the timed region
    with pinned_to_core0() as core:
        t0 = time.perf_counter()
        oracle.run(layers, [len(layers) - 1], [1], Bs, 1, p0, data, wl.optimizer, wl.lr)
        dt = time.perf_counter() - t0
    return {"value": scale * Bs / dt, "unit": "samples/s", "cores": 1, "kind": "oracle",
            "cpu_model": cpu_model(), "nproc": os.cpu_count(), "pinned_core": core,
            "sample": f"{text}; fwd+bwd+{'Adam' if wl.optimizer else 'SGD'}, single-threaded fp32 naive loops "
                      f"pinned to core {core} (taskset -c {core} equivalent), {dt:.1f} s"}


# ----------------------------------------------------------------------------- per-stage table

def solo_stage(plan, s, layers, wl, p0, data, n_data, M_solo, runs=3, warm=2, profile=True):
    """Stage s (replica 0) of `plan` alone on this GPU (pd_stage_solo: absent neighbours are
    infinitely fast stand-ins).  Returns ms per minibatch of this replica and kernel-class
    shares of an instrumented run."""
    import paper_conf_sosp_narayananhpsdgg19_b200 as pd
    from paper_conf_sosp_narayananhpsdgg19_b200.session import Pipeline, workers_of
    wid = [w for w, st, r, g in workers_of(plan) if st == s and r == 0][0]
    first, last, R = plan.stages[s][0], plan.stages[s][1], plan.stages[s][2]
    P = Pipeline(plan, layers, p0, dtype=pd.PD_BF16, optimizer=wl.optimizer, lr=wl.lr, minibatch=wl.batch,
                 record_trace=2, local=lambda w: w == wid, solo=True)
    try:
        P.set_data(*data, n_data)
        P.set_timing(2, 0)
        for _ in range(warm):
            P.run(M_solo)
        ms = []
        for _ in range(runs):
            P.run(M_solo)
            ms.append(P.stats()["run_ms"])
        mb = M_solo // R  # minibatches this replica processes per run
        out = {"stage": s, "layers": [first, last], "replicas": R, "ms_per_minibatch": float(np.median(ms)) / mb}
        if profile:
            P.set_timing(2, 0xFF)
            P.run(M_solo)
            st = P.stats()
            out["class_ms_per_minibatch"] = {k: st["kern_ms"][i] / mb for i, k in enumerate(pd.KERNEL_CLASSES)}
            out["instrumented_ms_per_minibatch"] = st["run_ms"] / mb
    finally:
        P.close()
    return out


def stage_table(args, wl, peaks, n_plan, only=-1):
    """Every stage of the n_plan-GPU plan bench.py would run, measured alone (solo mode); the
    slowest stage sets the pipeline's throughput (L775-777): projected = B * min_s R_s / t_s."""
    import synth
    layers, B = wl.layers, wl.batch
    plan = choose_plan(args.config, "pipeline", n_plan, layers, B, peaks)
    p0 = synth.init_params(layers)
    n_data = 8
    data = synth.make_data(wl, n_data)
    rows = []
    for s in range(len(plan.stages)):
        if only >= 0 and s != only:
            continue
        R = plan.stages[s][2]
        M_solo = 8 * int(np.lcm.reduce([st[2] for st in plan.stages]))  # pd_run: a multiple of every R_s
        quick = getattr(args, "solo_runs", 3) <= 1
        r = solo_stage(plan, s, layers, wl, p0, data, n_data, M_solo, runs=max(1, getattr(args, "solo_runs", 3)),
                       warm=1 if quick else 2, profile=not quick)
        r.setdefault("class_ms_per_minibatch", {})
        r["gflop_per_minibatch"] = sum(layer_flops(layers[l], B) * (2.0 / 3.0 if l == 0 else 1.0)
                                       for l in range(plan.stages[s][0], plan.stages[s][1] + 1)) / 1e9
        r["tflops"] = r["gflop_per_minibatch"] / r["ms_per_minibatch"]
        r["frac_sustained_peak"] = r["tflops"] / peaks["bf16_tflops_sustained"]
        rows.append(r)
        print(json.dumps({"solo_stage": r}), file=sys.stderr, flush=True)
    out = {"plan": [[a, b, r] for a, b, r, _g in plan.stages], "n_gpus": n_plan, "stages": rows,
           "method": "pd_stage_solo: each stage (replica 0) alone on one GPU, neighbours replaced by "
                     "infinitely fast stand-ins, receive rings synthetic; 3 timed runs of 8 R_s minibatches "
                     "after 2 warm-up runs, median"}
    if only < 0:
        slow = max(rows, key=lambda r: r["ms_per_minibatch"] / r["replicas"])
        proj = B * slow["replicas"] / (slow["ms_per_minibatch"] / 1e3)
        out.update({"slowest_stage": slow["stage"], "projected_samples_per_s": proj,
                    "projection": "B * R_s / t_s of the slowest stage (no transfer or bubble cost)"})
    return out


# ----------------------------------------------------------------------------- main arm

def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="gnmt16", choices=["mlp4096", "gnmt8", "gnmt16", "vgg16"])
    ap.add_argument("--minibatches", type=int, default=0,
                    help="minibatches per step (default 8 for one stage; 1024 for n > 1 stages: steady state, "
                         "fill/drain bubble (n-1)/(M+n-1) < 1 %%)")
    ap.add_argument("--stage-plan", type=int, default=-1,
                    help="per-stage table (solo mode, pd_stage_solo): each stage of the N-GPU plan measured "
                         "alone on this GPU, projected N-GPU throughput = B min_s R_s / t_s (L775-777); 0 = off; "
                         "default: the GPU count BASELINE.json names for the config (GNMT-16 8, GNMT-8 4, "
                         "MLP-4096 4, VGG-16 8 as 7-1)")
    ap.add_argument("--stage", type=int, default=-1,
                    help="measure only this stage of the --stage-plan plan in solo mode (for ncu) and exit")
    ap.add_argument("--solo-runs", type=int, default=3,
                    help="timed runs per stage in solo mode (1 = one warm-up + one run, no profile pass: for ncu)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--cpu-batch", type=int, default=0,
                    help="samples in the oracle's bounded sample (default: 8 for mlp4096, 1 otherwise -- ~10-60 s)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--plan", default="pipeline", choices=["pipeline", "dp"],
                    help="pipeline: pd_plan straight pipeline (VGG: (N-1)-1); dp: one stage x N replicas "
                         "(pure data parallelism, SURVEY §8(f) NEXT #1)")
    ap.add_argument("--sync", default="stash", choices=["stash", "vertical", "gpipe"],
                    help="weight stashing (default), vertical sync (§3.3; straight plans) or the GPipe "
                         "comparison schedule (§5.4: flush every NOAM minibatches, aggregated update)")
    args = ap.parse_args()
    if args.stage_plan < 0:
        args.stage_plan = {"gnmt16": 8, "gnmt8": 4, "mlp4096": 4, "vgg16": 8}[args.config]
    if args.cpu_batch <= 0:
        args.cpu_batch = 8 if args.config == "mlp4096" else 1
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist
    import synth
    if args.stage >= 0:  # one stage of the --stage-plan plan in solo mode (ncu captures), then exit
        wl = synth.workload(args.config)
        print(json.dumps(stage_table(args, wl, load_peaks(), args.stage_plan or 8, only=args.stage)), flush=True)
        return
    import paper_conf_sosp_narayananhpsdgg19_b200 as pd
    from paper_conf_sosp_narayananhpsdgg19_b200.session import Pipeline, stage_of_rank, torch_allgather

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    N = args.gpus
    if world != N:
        raise SystemExit(f"--gpus {N} but WORLD_SIZE {world}")
    torch.cuda.set_device(local_rank)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def allmax(x):
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def allsum(x):
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
        return float(t.item())

    peaks = load_peaks()
    wl = synth.workload(args.config)
    layers, B = wl.layers, wl.batch
    plan = choose_plan(args.config, args.plan, N, layers, B, peaks)
    n = len(plan.stages)
    R0 = plan.stages[0][2]
    M = args.minibatches or (8 * R0 if n == 1 else 1024)
    M = -(-M // R0) * R0  # a multiple of every replica count
    p0 = synth.init_params(layers) if True else None
    n_data = 8
    data = synth.make_data(wl, n_data)
    sync = {"stash": pd.PD_SYNC_STASH, "vertical": pd.PD_SYNC_VERTICAL, "gpipe": pd.PD_SYNC_GPIPE}[args.sync]
    P = Pipeline(plan, layers, p0, dtype=pd.PD_BF16, optimizer=wl.optimizer, lr=wl.lr, minibatch=B, sync_mode=sync,
                 record_trace=int(os.environ.get("PD_BENCH_TRACE", "2")), device_of=lambda g: g if world > 1 else local_rank,
                 local=(lambda wid: wid == rank) if world > 1 else None,
                 allgather=torch_allgather() if world > 1 else None)
    P.set_data(*data, n_data)
    clocks = Clocks(local_rank)
    clocks.start()  # sampled over warm-up + timed region (200 ms period)
    # timed region instrumentation: per-op CUDA events only (bubble, per-run span); per-kernel
    # events cannot live inside the CUDA graphs the runtime replays for launch-bound stages,
    # so kernel durations (roofline, step shares) come from a separate instrumented profile
    # pass right after the timed region, in this same run
    P.set_timing(2, 0)
    barrier()
    for _ in range(args.warmup):
        P.run(M)
    barrier()
    step_ms, launches, kern_ms, kern_cnt, bubbles = [], 0, np.zeros(8), np.zeros(8), []
    barrier()
    t_wall0 = time.perf_counter()
    for _ in range(args.steps):
        P.run(M)
        st = P.stats()
        step_ms.append(allmax(st["run_ms"]))
        launches += st["kernel_launches"]
        kern_ms += np.array(st["kern_ms"])
        kern_cnt += np.array(st["kern_count"])
        bubbles.append(st["bubble"])
    barrier()
    wall = time.perf_counter() - t_wall0
    clk = clocks.stop()
    total_ms = sum(step_ms)
    samples = args.steps * M * B
    value = samples / (total_ms / 1e3)
    launches = int(allsum(launches))
    bubble = allmax(float(np.mean(bubbles)))

    # ---- profile pass (not part of `value`): every kernel class timed, for step shares
    P.set_timing(2, 0xFF)
    prof_ms, prof_kern = 0.0, np.zeros(8)
    prof_cnt = np.zeros(8)
    for _ in range(2):
        P.run(M)
        st = P.stats()
        prof_ms += st["run_ms"]
        prof_kern += np.array(st["kern_ms"])
        prof_cnt += np.array(st["kern_count"])
    P.set_timing(2, 0)

    # ---- roofline of the dominant kernel, this rank's stage
    s_mine = stage_of_rank(plan, rank)
    first_l, last_l = plan.stages[s_mine][0], plan.stages[s_mine][1]
    my_layers = [layers[l] for l in range(first_l, last_l + 1)]
    lin = [L for L in my_layers if L.kind == synth.LINEAR] or my_layers
    stage_flops = sum(layer_flops(L, B) for L in my_layers)
    mb_mine = 2 * M // plan.stages[s_mine][2]  # minibatches of this replica in the profile pass
    cfl = class_flops(layers, first_l, last_l, B)  # per minibatch, per kernel class
    cls_s = prof_kern / 1e3
    cls_tflops = [cfl[i] * mb_mine / cls_s[i] / 1e12 if cls_s[i] > 0 and cfl[i] > 0 else 0.0 for i in range(8)]
    names = pd.KERNEL_CLASSES
    if args.config == "mlp4096":
        # HBM-bound: dW GEMM with the fused SGD update (K = 256), bytes per launch
        dw_avg_s = prof_kern[2] / max(prof_cnt[2], 1) / 1e3
        dw_bytes = float(np.mean([dw_update_bytes(L, B) for L in lin]))
        achieved = dw_bytes / dw_avg_s / 1e9 if dw_avg_s > 0 else 0.0
        roof = {"bound": "hbm", "kernel": "dW GEMM + fused SGD update (tcgen05, EPI_SGD)",
                "achieved": achieved, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                "frac": achieved / peaks["hbm_gbs"], "traffic": ncu_traffic("dw_update_sgd", args.config),
                "traffic_source": "ncu --set full capture of one launch (profiles/ncu_traffic_r*.json); "
                                  "writes still dirty in L2 at kernel end are not in dram__bytes_write",
                "bytes_per_launch": dw_bytes, "avg_launch_us": dw_avg_s * 1e6,
                "peak_source": peaks["source"] + " hbm_gbs (copy)"}
    else:
        # tensor-bound stages: the kernel class with the largest share of the step
        d = int(np.argmax([cls_s[i] if cfl[i] > 0 else 0.0 for i in range(8)]))
        avg_s = prof_kern[d] / max(prof_cnt[d], 1) / 1e3
        per_launch = cfl[d] * mb_mine / max(prof_cnt[d], 1)
        roof = {"bound": "tensor", "kernel": names[d], "achieved": cls_tflops[d],
                "peak": peaks["bf16_tflops_sustained"], "unit": "TFLOP/s",
                "frac": cls_tflops[d] / peaks["bf16_tflops_sustained"],
                "traffic": ncu_traffic(names[d], args.config),
                "flops_per_launch": per_launch, "avg_launch_us": avg_s * 1e6,
                "flops_per_minibatch": cfl[d],
                "peak_source": peaks["source"] + " bf16_tflops_sustained (cuBLAS)"}
        if roof["traffic"] and avg_s > 0:
            # the same launch against the memory roof: DRAM bytes of one launch (ncu --set full)
            # over its live average duration -- a wavefront kernel re-streams every layer's
            # weights once per wave (they exceed the on-chip capacity at N = 1), so it is bound
            # by HBM / per-SM ingest, not by the tensor pipe
            gbs = roof["traffic"] / avg_s / 1e9
            roof["memory_view"] = {"dram_gbs": gbs, "frac_hbm": gbs / peaks["hbm_gbs"],
                                   "hbm_peak_gbs": peaks["hbm_gbs"],
                                   "note": "ncu dram__bytes_read+write per launch / live avg launch time"}
    fw_tflops, dx_tflops, dw_tflops = cls_tflops[0], cls_tflops[1], cls_tflops[2]
    step_share = {cls: float(prof_kern[i] / max(prof_ms, 1e-9)) for i, cls in enumerate(names)}
    step_share["note"] = "profile pass (2 steps, every kernel class event-timed); dW and dX overlap on two streams"

    # ---- end to end through the public API: host (pinned) inputs in, losses out, every step
    e2e = None
    if not args.no_e2e:
        inputs, tokens, labels = data
        src = tokens if inputs is None else inputs
        pin_in = torch.from_numpy(np.ascontiguousarray(np.resize(src, (M,) + src.shape[1:]))).pin_memory()
        pin_lab = torch.from_numpy(np.ascontiguousarray(np.resize(labels, (M,) + labels.shape[1:]))).pin_memory()
        tok_arg = pin_in if inputs is None else None
        in_arg = None if inputs is None else pin_in
        P.set_data(in_arg, tok_arg, pin_lab, M)
        P.run(M)  # warm the M-sized data ring
        barrier()
        t0 = time.perf_counter()
        for _ in range(args.steps):
            P.set_data(in_arg, tok_arg, pin_lab, M)
            P.run(M)
            P.losses(M)
        barrier()
        e2e_s = allmax(time.perf_counter() - t0)
        e2e = {"value": samples / e2e_s, "unit": "samples/s",
               "h2d_bytes_per_step": int(pin_in.numel() * 4 + pin_lab.numel() * 4) if s_mine in (0, n - 1) else 0,
               "d2h_bytes_per_step": int(M * 4),
               "note": "wall clock around set_data(pinned host) + pd_run + pd_get_losses, max over ranks"}

    roof_sps, roof_slow, roof_stages = stage_roofline(layers, plan, B, peaks, wl.optimizer)
    P.close()
    cpu = None
    if rank == 0 and N == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(args, layers, wl)
    solo = None
    if rank == 0 and N == 1 and args.stage_plan > 1:
        solo = stage_table(args, wl, peaks, args.stage_plan)
        solo["projected_speedup_over_this_run"] = solo["projected_samples_per_s"] / value
    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "samples/s", "n_gpus": N, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": total_ms / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "bf16", "data": "synthetic",
            "config": {"workload": WORKLOAD_DESC.get(args.config, args.config) +
                                   f", minibatch {B}, bf16 weights/activations, fp32 master, "
                                   f"{'Adam' if wl.optimizer else 'SGD'} lr {wl.lr}",
                       "plan": "-".join(str(s[2]) for s in plan.stages) + f" ({n} stage{'s' if n > 1 else ''} "
                               f"of {[s[1] - s[0] + 1 for s in plan.stages]} layers)",
                       "global_batch": B, "minibatches_per_step": M, "noam": plan.noam,
                       "parallelism": (f"pipeline{n}" if n > 1 else
                                       (f"dp{N}" if N > 1 else "single-stage")),
                       "sync": args.sync,
                       "l2": l2_note(layers, wl.optimizer)},
            "bubble_pct": 100.0 * bubble,
            "wall_s": wall,
            "gpu_launches": launches,
            "clocks": clk,
            "roofline": dict(roof, timing="CUDA events around every launch of the class on its stream, "
                                          "instrumented profile pass (2 steps) right after the timed region; "
                                          "dW overlaps the next layer's dX"),
            "tensor_pipe": {"class_tflops": {n: t for n, t in zip(pd.KERNEL_CLASSES, cls_tflops) if t > 0},
                            "class_frac": {n: t / peaks["bf16_tflops_sustained"]
                                           for n, t in zip(pd.KERNEL_CLASSES, cls_tflops) if t > 0},
                            "peak_tflops": peaks["bf16_tflops_sustained"],
                            "note": "algorithmic class FLOPs (bench.class_flops) / class device time (CUDA events, "
                                    "profile pass); dW time includes a fused update; ncu tensor-pipe counters "
                                    "per stage are in profiles/",
                            "peak_source": peaks["source"] + " bf16_tflops_sustained (cuBLAS)"},
            "step_share": step_share,
            "stage_tflops": stage_flops * args.steps * M / plan.stages[s_mine][2] / (total_ms / 1e3) / 1e12,
            "pipeline_roofline": {"samples_per_s": roof_sps, "frac": value / roof_sps, "slowest_stage": roof_slow,
                                  "stages": roof_stages,
                                  "definition": "B * min_s R_s / max(F_s/P_tensor_sustained, H_s/BW_HBM, "
                                                "N_s/900 GB/s) (north_star; bench.stage_roofline)"},
            "e2e": e2e,
            "cpu_baseline": cpu,
            "stage_table": solo,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
