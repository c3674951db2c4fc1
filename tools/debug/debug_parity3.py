import sys, os
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", "..", "tests"))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import numpy as np
import synth, torchref
import paper_conf_sosp_narayananhpsdgg19_b200 as pd
from gpu_helpers import run_both
wl = synth.workload("mlp4096", reduced=True)
for M in [2, 2, 4, 2, 6]:
    res = run_both(wl, [15], [2], M, pd.PD_FP32)
    print(M, "losses", np.round(res["losses"], 5), "ref", np.round(res["ref"].losses, 5),
          "perr", torchref.max_rel_err(res["got"], res["ref"].params), flush=True)
