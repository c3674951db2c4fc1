"""Persistent LSTM recurrence kernels (csrc/lstm_rec.cu) against the oracle.

The reduced GNMT configs (H = 32) run the per-step path; these GNMT-shaped stacks have
H % 256 == 0, so the bf16 path runs each layer's whole recurrence (forward and
backward-through-time) as one persistent launch.  SGD makes the parameter deltas a direct
image of the gradients, so a wrong step, a wrong K-range or a mis-ordered partial shows up in
the delta error; losses check the forward pass minibatch by minibatch.  The same run with
PD_LSTM_REC=0 (per-step GEMM + cell kernels) must agree with it closely."""
import os

import numpy as np
import pytest

import synth
import torchref
import paper_conf_sosp_narayananhpsdgg19_b200 as pd
from gpu_helpers import run_both, assert_schedule_exact, param_errors, BF16_TOL

pytestmark = pytest.mark.gpu

# (layers, H, B, T): ragged batch (N = 48 > B = 40), full GNMT width with one and two layers.
# One layer runs the persistent per-layer kernels; runs of >= 2 layers the wavefront kernel
# (lstm_wave.cu) unless PD_LSTM_WAVE=0.
SHAPES = [(2, 256, 16, 6), (1, 512, 40, 5), (1, 1024, 64, 4), (2, 1024, 64, 3)]
WAVE_SHAPES = [(4, 256, 16, 6), (3, 512, 40, 5), (8, 128, 8, 4), (4, 1024, 64, 3), (3, 1024, 64, 3)]


def _workload(n, H, B, T):
    return synth.Workload(f"lstm{n}x{H}", synth.gnmt(n, H, 512, T, B), B, synth.SGD, 0.05)


def _run(wl, last, M, rec, wave=True):
    old = {k: os.environ.get(k) for k in ("PD_LSTM_REC", "PD_LSTM_WAVE")}
    os.environ["PD_LSTM_REC"] = "1" if rec else "0"
    os.environ["PD_LSTM_WAVE"] = "1" if wave else "0"
    try:
        return run_both(wl, last, [1] * len(last), M, pd.PD_BF16, n_data=3)
    finally:
        for k, v in old.items():
            if v is None:
                del os.environ[k]
            else:
                os.environ[k] = v


@pytest.mark.parametrize("n,H,B,T", SHAPES)
def test_persistent_recurrence_matches_oracle(n, H, B, T):
    wl = _workload(n, H, B, T)
    M = 3
    res = _run(wl, [len(wl.layers) - 1], M, rec=True)
    assert_schedule_exact(res)
    perr, derr = param_errors(res)
    assert perr < BF16_TOL, perr
    assert derr < 5e-2, derr
    np.testing.assert_allclose(res["losses"], res["ref"].losses, rtol=1e-2)


@pytest.mark.parametrize("n,H,B,T", SHAPES[:3])
def test_persistent_equals_per_step_path(n, H, B, T):
    wl = _workload(n, H, B, T)
    a = _run(wl, [len(wl.layers) - 1], 2, rec=True)
    b = _run(wl, [len(wl.layers) - 1], 2, rec=False)
    # same bf16 operands and roundings except the fp32 summation order of the recurrent GEMM
    d = torchref.delta_err(a["got"], b["got"], a["p0"])
    assert d < 2e-2, d
    np.testing.assert_allclose(a["losses"], b["losses"], rtol=2e-3)


def test_persistent_two_stage_pipeline_only_first_worker_lstm():
    # stage 0 = Emb + LSTM (persistent: the only LSTM worker on the GPU), stage 1 = classifier
    wl = _workload(1, 256, 16, 5)
    res = _run(wl, [1, 2], 8, rec=True)
    assert_schedule_exact(res)
    perr, derr = param_errors(res)
    assert perr < BF16_TOL and derr < 5e-2, (perr, derr)


@pytest.mark.parametrize("n,H,B,T", WAVE_SHAPES)
def test_wavefront_matches_oracle(n, H, B, T):
    wl = _workload(n, H, B, T)
    res = _run(wl, [len(wl.layers) - 1], 3, rec=True)
    assert_schedule_exact(res)
    perr, derr = param_errors(res)
    assert perr < BF16_TOL, perr
    assert derr < 5e-2, derr
    np.testing.assert_allclose(res["losses"], res["ref"].losses, rtol=1e-2)


@pytest.mark.parametrize("n,H,B,T", WAVE_SHAPES[:2])
def test_wavefront_equals_per_layer_kernels(n, H, B, T):
    wl = _workload(n, H, B, T)
    a = _run(wl, [len(wl.layers) - 1], 2, rec=True, wave=True)
    b = _run(wl, [len(wl.layers) - 1], 2, rec=True, wave=False)
    d = torchref.delta_err(a["got"], b["got"], a["p0"])
    assert d < 2e-2, d
    np.testing.assert_allclose(a["losses"], b["losses"], rtol=2e-3)


def test_wavefront_inside_a_pipeline_stage():
    # stage 0 = Emb + 3 LSTMs (one wavefront run, dX of the bottom layer into the embedding),
    # stage 1 = classifier: startup / steady state / drain with stashed versions
    wl = _workload(3, 256, 16, 5)
    res = _run(wl, [3, 4], 8, rec=True)
    assert_schedule_exact(res)
    perr, derr = param_errors(res)
    assert perr < BF16_TOL and derr < 5e-2, (perr, derr)


def _run_env(wl, last, M, env):
    old = {k: os.environ.get(k) for k in env}
    os.environ.update(env)
    try:
        return run_both(wl, last, [1] * len(last), M, pd.PD_BF16, n_data=3)
    finally:
        for k, v in old.items():
            if v is None:
                del os.environ[k]
            else:
                os.environ[k] = v


@pytest.mark.parametrize("opt", [synth.SGD, synth.ADAM])
def test_split_weight_gradient_path_matches_oracle(opt):
    # PD_DW_SPLIT_K: the long-K weight gradients (LSTM W_ih/W_hh over T*B rows, classifier) as
    # 2-CTA GEMM -> fp32 gradient -> vectorised update, instead of the fused-epilogue GEMM;
    # (4, 256, 16, 6): M = 4H = 1024, N = 256, K = 96 / 80; classifier M = 512, N = 256, K = 96
    wl = synth.Workload("lstm4x256", synth.gnmt(4, 256, 512, 6, 16), 16, opt, 0.05 if opt == synth.SGD else 3e-4)
    last = [len(wl.layers) - 1]
    a = _run_env(wl, last, 3, {"PD_DW_SPLIT_K": "64"})
    assert_schedule_exact(a)
    perr, derr = param_errors(a)
    assert perr < BF16_TOL, perr
    if opt == synth.SGD:
        assert derr < 5e-2, derr
    b = _run_env(wl, last, 3, {"PD_DW_SPLIT_K": "0"})
    # same bf16 operands; only the GEMM tiling (fp32 summation order) and the update kernel differ
    if opt == synth.SGD:
        d = torchref.delta_err(a["got"], b["got"], a["p0"])
        assert d < 2e-2, d
    else:  # Adam moves every weight by ~lr*sign(g): compare parameters, not deltas
        assert torchref.max_rel_err(a["got"], b["got"]) < 2e-2
    np.testing.assert_allclose(a["losses"], b["losses"], rtol=2e-3)


# Weight gradients of a short wavefront run computed on the idle SMs WHILE the backward wave
# runs (runtime wave_dw_overlap: chunks of 10 timesteps, last first, each waiting for the
# wave's step counter; reduce-added fp32 partials): against the oracle, and against the
# gradients computed after the wave (PD_WAVE_DW=0) -- equal up to the fp32 order of the chunk
# sums.  (3, 512, 32, 21): 3 chunks per GEMM; (2, 256, 40, 23): chunk boundaries inside a
# 64-row K-block (B = 40).
@pytest.mark.parametrize("n,H,B,T", [(3, 512, 32, 21), (2, 256, 40, 23)])
def test_wave_weight_gradients_overlapped(n, H, B, T):
    wl = _workload(n, H, B, T)
    last = [len(wl.layers) - 1]
    a = _run_env(wl, last, 2, {"PD_LSTM_REC": "1", "PD_LSTM_WAVE": "1", "PD_WAVE_DW": "1"})
    b = _run_env(wl, last, 2, {"PD_LSTM_REC": "1", "PD_LSTM_WAVE": "1", "PD_WAVE_DW": "0"})
    assert_schedule_exact(a)
    perr, derr = param_errors(a)
    assert perr < BF16_TOL and derr < 5e-2, (perr, derr)
    d = torchref.delta_err(a["got"], b["got"], a["p0"])
    assert d < 1e-2, d
    np.testing.assert_allclose(a["losses"], b["losses"], rtol=1e-5)
