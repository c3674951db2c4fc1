"""Per-layer parity diagnostics (GPU): prints param / delta errors per layer vs the oracle."""
import sys, os
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", "..", "tests"))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import numpy as np
import synth
import paper_conf_sosp_narayananhpsdgg19_b200 as pd
from gpu_helpers import run_both

def show(name, wl, last, reps, M, dtype, lr=None):
    res = run_both(wl, last, reps, M, dtype, lr=lr)
    print(f"== {name}")
    for l, (g, r, i) in enumerate(zip(res["got"], res["ref"].params, res["p0"])):
        if r.size == 0: continue
        pe = np.abs(g - r).max() / np.abs(r).max()
        d = np.abs(r - i).max()
        de = np.abs((g - i) - (r - i)).max() / max(d, 1e-30)
        print(f"  layer {l:2d} param_err {pe:.2e} delta {d:.2e} delta_err {de:.2e} nan={np.isnan(g).any()}")

wl = synth.workload("mlp4096", reduced=True)
show("fp32 [4] single stage", wl, [15], [4], 8, pd.PD_FP32)
show("fp32 [2] single stage", wl, [15], [2], 8, pd.PD_FP32)
show("fp32 [1,1] ", wl, [7, 15], [1, 1], 8, pd.PD_FP32)
show("bf16 [1] single", wl, [15], [1], 8, pd.PD_BF16)
show("bf16 [1] single lr .05", wl, [15], [1], 8, pd.PD_BF16, lr=0.05)
show("bf16 4-stage", wl, [3, 7, 11, 15], [1]*4, 16, pd.PD_BF16)
