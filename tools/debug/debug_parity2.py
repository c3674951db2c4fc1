import sys, os
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", "..", "tests"))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import numpy as np
import synth
import paper_conf_sosp_narayananhpsdgg19_b200 as pd
from gpu_helpers import run_both

def show(name, wl, last, reps, M, dtype, lr=None):
    res = run_both(wl, last, reps, M, dtype, lr=lr)
    print(f"== {name}  losses gpu {np.round(res['losses'][:4],5)} ref {np.round(res['ref'].losses[:4],5)}")
    for l, (g, r, i) in enumerate(zip(res["got"], res["ref"].params, res["p0"])):
        if r.size == 0: continue
        L = wl.layers[l]
        nW = L.out * L.in_
        d = np.abs(r - i).max()
        de = np.abs((g - i) - (r - i)).max() / max(d, 1e-30)
        dW = np.abs((g[:nW]-i[:nW]) - (r[:nW]-i[:nW])).max() / max(np.abs(r[:nW]-i[:nW]).max(), 1e-30)
        db = np.abs((g[nW:]-i[nW:]) - (r[nW:]-i[nW:])).max() / max(np.abs(r[nW:]-i[nW:]).max(), 1e-30)
        print(f"  layer {l:2d} delta {d:.2e} delta_err {de:.2e} (W {dW:.2e} b {db:.2e})")

wl = synth.workload("mlp4096", reduced=True)
show("fp32 [2] M=2", wl, [15], [2], 2, pd.PD_FP32)
show("fp32 [2] M=4", wl, [15], [2], 4, pd.PD_FP32)
show("fp32 [2,1] M=4", wl, [7, 15], [2, 1], 4, pd.PD_FP32)
show("bf16 [1] M=1", wl, [15], [1], 1, pd.PD_BF16)
show("bf16 [1] M=1 lr .05", wl, [15], [1], 1, pd.PD_BF16, lr=0.05)
