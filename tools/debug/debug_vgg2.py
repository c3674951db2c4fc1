import sys, os, copy
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", "..", "tests"))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import numpy as np
import synth, torchref
import paper_conf_sosp_narayananhpsdgg19_b200 as pd
from gpu_helpers import run_both
wlb = synth.Workload("vgg_r16", synth.vgg([[8], [16]], 8, 3, [32], 16), 4, synth.SGD, 0.05)
for lr in [0.05, 0.005, 0.0005]:
    for M in [1, 2, 3, 5]:
        res = run_both(wlb, [5], [1], M, pd.PD_BF16, lr=lr)
        pe = torchref.max_rel_err(res["got"], res["ref"].params)
        de = torchref.delta_err(res["got"], res["ref"].params, res["p0"])
        per = [float(np.abs((g-i)-(r-i)).max()/max(np.abs(r-i).max(),1e-30)) for g, r, i in zip(res["got"], res["ref"].params, res["p0"]) if r.size]
        print(f"lr {lr} M {M} perr {pe:.2e} derr {de:.2e} per-layer {np.round(per,3)}", flush=True)
