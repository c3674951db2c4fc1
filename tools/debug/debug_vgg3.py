import sys, os, copy
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", "..", "tests"))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import numpy as np
import synth, torchref
import paper_conf_sosp_narayananhpsdgg19_b200 as pd
from gpu_helpers import run_both
cases = {
 "c64": synth.vgg([[64]], 16, 8, [], 16),
 "c64x2": synth.vgg([[64, 64]], 16, 8, [], 16),
 "c3_64": synth.vgg([[64]], 16, 3, [], 16),
 "c64_128": synth.vgg([[64], [128]], 16, 8, [], 16),
 "full": synth.vgg([[64, 64], [128]], 16, 3, [64], 16),
}
for name, layers in cases.items():
    wl = synth.Workload(name, layers, 8, synth.SGD, 0.02)
    for dt in (pd.PD_FP32, pd.PD_BF16):
        res = run_both(wl, [len(layers) - 1], [1], 1, dt, n_data=2)
        per = [float(np.abs((g-i)-(r-i)).max()/max(np.abs(r-i).max(),1e-30)) for g, r, i in zip(res["got"], res["ref"].params, res["p0"]) if r.size]
        print(f"{name} dt {dt} loss {res['losses'][0]:.5f} ref {res['ref'].losses[0]:.5f} per-layer delta err {np.round(per,4)}", flush=True)
