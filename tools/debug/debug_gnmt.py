import sys, os
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", "..", "tests"))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import numpy as np
import synth
import paper_conf_sosp_narayananhpsdgg19_b200 as pd
from gpu_helpers import run_both
wl = synth.workload("gnmt8", reduced=True)
for dtype in (pd.PD_FP32, pd.PD_BF16):
    for last, reps, M in [([9], [1], 1), ([9], [1], 3), ([4, 9], [1, 1], 8)]:
        try:
            res = run_both(wl, last, reps, M, dtype)
        except Exception as e:
            print("ERR", dtype, last, e); continue
        print(f"== dtype {dtype} plan {last} M {M} losses {np.round(res['losses'][:3],5)} ref {np.round(res['ref'].losses[:3],5)}")
        for l, (g, r, i) in enumerate(zip(res["got"], res["ref"].params, res["p0"])):
            d = np.abs(r - i).max()
            print(f"  layer {l} kind {wl.layers[l].kind} perr {np.abs(g-r).max()/np.abs(r).max():.2e} delta {d:.2e} derr {np.abs((g-i)-(r-i)).max()/max(d,1e-30):.2e}")
