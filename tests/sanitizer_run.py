"""A small 2-stage bf16 pipeline (4 x Linear(256), stages [0,1 | 2,3], 8 minibatches) for the
compute-sanitizer runs of test_gpu_sanitizer.py; exits 0 when the trace matches the oracle."""
import os
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, HERE)
sys.path.insert(0, os.path.dirname(HERE))

import synth  # noqa: E402
import paper_conf_sosp_narayananhpsdgg19_b200 as pd  # noqa: E402
from gpu_helpers import run_both  # noqa: E402

if __name__ == "__main__":
    wl = synth.Workload("mlp256", synth.mlp([256] * 5, 64), 64, synth.SGD, 0.5)
    res = run_both(wl, [1, 3], [1, 1], 8, pd.PD_BF16, n_data=2)
    got = [t[:8] for t in res["trace"]]
    print("trace exact:", got == res["ref"].events)
    sys.exit(0 if got == res["ref"].events else 1)
