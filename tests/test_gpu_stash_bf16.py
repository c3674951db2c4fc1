"""bf16 weight-stashing parity that can fail on a version error, with negative controls
(VERDICT r1 "next round" #1; PAPER.md L1141-1161 stashing, L1227-1241 update rule,
L1349-1353 version lifetime).

* test_bf16_stash_discriminates: every case of stash_cases.py must land within 1/4 of the
  no-stash mutant's delta error of the stashing oracle and outside it for the no-stash
  oracle, with the event trace exact.
* test_fault_*: the same runs through fault-injected builds of the runtime (build.py FAULTS,
  loaded in a subprocess through PD_LIBRARY) must FAIL: a backward reading the latest
  instead of the stashed slot, a side-stream dW + update not ordered after dX / the
  gradient, and activation receive rings one slot too shallow (caught by the host
  slot-ownership checker before anything is overwritten).
"""
import json
import os
import subprocess
import sys

import pytest

import stash_cases
from paper_conf_sosp_narayananhpsdgg19_b200 import build as pdbuild

pytestmark = pytest.mark.gpu

HERE = os.path.dirname(os.path.abspath(__file__))


@pytest.mark.parametrize("name", stash_cases.CASES)
def test_bf16_stash_discriminates(name):
    r = stash_cases.evaluate(name)
    print(r)
    assert r["trace_exact"], r
    assert r["mutant_l2"] > 0.04, r  # the case makes stashing visible at all
    assert stash_cases.discriminates(r), r


def test_bf16_single_layer_first_stage():
    """Stage 0 = one Linear layer: its overlapped backward has no dX, so only the fork event
    orders the side stream's dW + update after the gradient arrives."""
    import numpy as np
    import paper_conf_sosp_narayananhpsdgg19_b200 as pd
    from gpu_helpers import run_both, assert_schedule_exact, param_errors, BF16_TOL
    wl, last, reps, M = stash_cases.case("mlp256_first1")
    res = run_both(wl, last, reps, M, pd.PD_BF16, n_data=4)
    assert_schedule_exact(res)
    perr, derr = param_errors(res)
    assert perr < BF16_TOL, (perr, derr)
    np.testing.assert_allclose(res["losses"], res["ref"].losses, rtol=2e-2)


def _run_faulty(fault, name):
    pdbuild.build_faults()
    env = dict(os.environ, PD_LIBRARY=pdbuild.fault_lib(fault))
    p = subprocess.run([sys.executable, os.path.join(HERE, "stash_cases.py"), name], env=env, capture_output=True,
                       text=True, timeout=600)
    lines = [ln for ln in p.stdout.splitlines() if ln.startswith("{")]
    assert lines, (p.returncode, p.stdout[-2000:], p.stderr[-2000:])
    return json.loads(lines[-1])


@pytest.mark.parametrize("name", ["mlp256", "gnmt_adam", "vgg"])
def test_fault_backward_reads_latest_version(name):
    r = _run_faulty("fault_stash", name)
    print(r)
    assert "error" in r or not r["discriminates"], r


@pytest.mark.parametrize("name", ["mlp256", "mlp256_first1"])
def test_fault_side_stream_unordered(name):
    r = _run_faulty("fault_no_dxwait", name)
    print(r)
    if name == "mlp256_first1":  # no stash effect at stage 0: the parity tolerance is the bar
        assert "error" in r or r["param_err"] > 2e-2, r
    else:
        assert "error" in r or not r["discriminates"], r


def test_fault_receive_ring_too_shallow():
    r = _run_faulty("fault_recv_depth", "mlp256")
    print(r)
    assert "error" in r and "slot ownership" in r["error"], r
