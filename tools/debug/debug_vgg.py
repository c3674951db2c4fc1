import sys, os
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", "..", "tests"))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import numpy as np
import synth
import paper_conf_sosp_narayananhpsdgg19_b200 as pd
from gpu_helpers import run_both
wl = synth.workload("vgg16", reduced=True)
wlb = synth.Workload("vgg_r16", synth.vgg([[8], [16]], 8, 3, [32], 16), 4, synth.SGD, 0.05)
for name, w, dtype in [("fp32", wl, pd.PD_FP32), ("bf16", wlb, pd.PD_BF16)]:
    for last, reps, M in [([5], [1], 1), ([5], [1], 3), ([2, 5], [1, 1], 6)]:
        try:
            res = run_both(w, last, reps, M, dtype)
        except Exception as e:
            print("ERR", name, last, repr(e)); continue
        print(f"== {name} plan {last} M {M} losses {np.round(res['losses'][:3],5)} ref {np.round(res['ref'].losses[:3],5)}", flush=True)
        for l, (g, r, i) in enumerate(zip(res["got"], res["ref"].params, res["p0"])):
            if r.size == 0: continue
            d = np.abs(r - i).max()
            print(f"  layer {l} kind {w.layers[l].kind} perr {np.abs(g-r).max()/np.abs(r).max():.2e} delta {d:.2e} derr {np.abs((g-i)-(r-i)).max()/max(d,1e-30):.2e}")
