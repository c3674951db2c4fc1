"""GPipe-style flush schedule with gradient aggregation on the B200 (PD_SYNC_GPIPE; PAPER.md
§5.4; R27): event trace and version map
bit-exact against the oracle's GPipe mode, parameters within the north-star tolerance, and a
discriminating bf16 case in which the 1F1B + stashing result is far from the GPipe one."""
import numpy as np
import pytest

import oracle
import synth
import paper_conf_sosp_narayananhpsdgg19_b200 as pd
from gpu_helpers import run_both, assert_schedule_exact, param_errors, FP32_TOL, BF16_TOL
from stash_cases import rel_l2

pytestmark = pytest.mark.gpu
GP = pd.PD_SYNC_GPIPE


@pytest.mark.parametrize("last,M,D", [([7, 15], 8, 0), ([3, 7, 11, 15], 16, 0), ([3, 7, 11, 15], 12, 3),
                                      ([0, 1, 2, 15], 8, 2), ([15], 6, 3), ([3, 7, 11, 15], 10, 5)])
def test_gpipe_mlp_fp32(last, M, D):
    wl = synth.workload("mlp4096", reduced=True)
    res = run_both(wl, last, [1] * len(last), M, pd.PD_FP32, noam=D, sync_mode=GP)
    assert_schedule_exact(res)
    Dg = D or len(last)
    assert (res["vmap"] == np.array([[t // Dg for t in range(M)]] * len(last))).all()
    perr, derr = param_errors(res)
    assert perr < FP32_TOL and derr < 1e-3, (perr, derr)
    assert np.allclose(res["losses"], res["ref"].losses, rtol=1e-4, atol=1e-5)


def test_gpipe_gnmt_fp32():
    wl = synth.workload("gnmt8", reduced=True)
    res = run_both(wl, [2, 5, 8, 9], [1] * 4, 16, pd.PD_FP32, sync_mode=GP)
    assert_schedule_exact(res)
    perr, derr = param_errors(res)
    assert perr < FP32_TOL and derr < 1e-3, (perr, derr)


def test_gpipe_vgg_fp32():
    wl = synth.workload("vgg16", reduced=True)
    res = run_both(wl, [2, 5], [1, 1], 8, pd.PD_FP32, sync_mode=GP)
    assert_schedule_exact(res)
    perr, derr = param_errors(res)
    assert perr < FP32_TOL and derr < 1e-3, (perr, derr)


def test_gpipe_bf16_all_kinds():
    wl = synth.workload("mlp4096", reduced=True)
    res = run_both(wl, [3, 7, 11, 15], [1] * 4, 16, pd.PD_BF16, lr=0.05, sync_mode=GP)
    assert_schedule_exact(res)
    assert param_errors(res)[0] < BF16_TOL
    g = synth.workload("gnmt8", reduced=True)
    res = run_both(g, [4, 9], [1, 1], 8, pd.PD_BF16, lr=3e-4, sync_mode=GP)
    assert_schedule_exact(res)
    assert param_errors(res)[0] < BF16_TOL
    v = synth.Workload("vgg_r16", synth.vgg([[8], [16]], 8, 3, [32], 16), 4, synth.SGD, 0.01)
    res = run_both(v, [2, 5], [1, 1], 8, pd.PD_BF16, sync_mode=GP)
    assert_schedule_exact(res)
    assert param_errors(res)[0] < BF16_TOL


def test_gpipe_bf16_discriminates_the_schedule():
    # 4 x Linear(256), 4 single-layer stages, SGD lr 2 (tests/stash_cases.py "mlp256"): here
    # 1F1B + weight stashing and GPipe's group-mean updates end far apart, so a bf16 run that
    # mixed them up (a per-minibatch update, a wrong group version) fails the rel-L2 bar
    wl = synth.Workload("mlp256", synth.mlp([256] * 5, 64), 64, synth.SGD, 2.0)
    last, M = [0, 1, 2, 3], 16
    res = run_both(wl, last, [1] * 4, M, pd.PD_BF16, n_data=4, sync_mode=GP)
    assert_schedule_exact(res)
    ref = res["ref"]
    other = oracle.run(wl.layers, last, [1] * 4, wl.batch, M, res["p0"], synth.make_data(wl, 4), wl.optimizer,
                       wl.lr)
    # distances relative to the GPipe trajectory's delta: the 1F1B oracle is `gap` away, the
    # run must be within gap/4 (so, by the triangle inequality, >= 3 gap/4 from 1F1B's)
    gap = rel_l2(other.params, ref.params, res["p0"])
    assert gap > 1.0, gap
    assert rel_l2(res["got"], ref.params, res["p0"]) <= gap / 4, gap


def test_gpipe_second_run_continues():
    # two pd_runs of M (groups never straddle a run) == one oracle run of 2M on data t mod 4
    from paper_conf_sosp_narayananhpsdgg19_b200.session import Pipeline
    wl = synth.workload("mlp4096", reduced=True)
    p0 = synth.init_params(wl.layers)
    data = synth.make_data(wl, 4)
    last, M = [3, 7, 11, 15], 8
    with Pipeline(pd.Plan.manual(last, [1] * 4), wl.layers, p0, dtype=pd.PD_FP32, lr=wl.lr,
                  minibatch=wl.batch, sync_mode=GP) as P:
        P.set_data(*data, 4)
        P.run(M)
        P.run(M)
        got = P.params([synth.param_count(L) for L in wl.layers])
        got = [got[l] for l in range(len(wl.layers))]
    ref = oracle.run(wl.layers, last, [1] * 4, wl.batch, 2 * M, p0, data, wl.optimizer, wl.lr, gpipe=True)
    import torchref
    assert torchref.max_rel_err(got, ref.params) < FP32_TOL


def test_gpipe_bubble_exceeds_1f1b():
    # the flush every D minibatches: measured busy fraction of the workers below 1F1B's on the
    # same plan (both on one GPU's streams; §5.4 attributes GPipe's slowdown to the flushes)
    wl = synth.workload("mlp4096", reduced=True)
    last, M = [3, 7, 11, 15], 32
    b = {}
    for mode in (pd.PD_SYNC_STASH, GP):
        res = run_both(wl, last, [1] * 4, M, pd.PD_FP32, sync_mode=mode, record_trace=2)
        b[mode] = res["stats"]["bubble"]
    assert b[GP] > b[pd.PD_SYNC_STASH], b
