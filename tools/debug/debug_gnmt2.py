import sys, os
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", "..", "tests"))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import numpy as np, copy
import synth, torchref
import paper_conf_sosp_narayananhpsdgg19_b200 as pd
from gpu_helpers import run_both
base = synth.workload("gnmt8", reduced=True)
for opt, lr in [(synth.SGD, 0.05), (synth.SGD, 0.5), (synth.ADAM, 3e-4), (synth.ADAM, 1e-3)]:
    wl = copy.copy(base); wl.optimizer = opt; wl.lr = lr
    res = run_both(wl, [4, 9], [1, 1], 8, pd.PD_BF16)
    pe = torchref.max_rel_err(res["got"], res["ref"].params)
    de = torchref.delta_err(res["got"], res["ref"].params, res["p0"])
    # fraction of elements whose delta sign disagrees
    flips = np.mean(np.concatenate([np.sign(g - i) != np.sign(r - i) for g, r, i in zip(res["got"], res["ref"].params, res["p0"])]))
    print(f"opt {opt} lr {lr}: perr {pe:.3e} derr {de:.3e} sign-flip frac {flips:.4f}", flush=True)
