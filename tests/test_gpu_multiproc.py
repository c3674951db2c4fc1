"""One process per worker (the bench/torchrun layout) on ONE B200: two processes share
cuda:0, exchange CUDA-IPC blobs over torch.distributed (gloo), and synchronise only through
the flag words + cuStreamWaitValue32 path.  Trace, version map and parameters must match
the oracle exactly as in the single-process case."""
import os
import pickle
import socket
import tempfile

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, stage_last, reps, dtype, M, out_dir, runs=1):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch.distributed as dist
    import synth
    import paper_conf_sosp_narayananhpsdgg19_b200 as pd
    from paper_conf_sosp_narayananhpsdgg19_b200.session import Pipeline, torch_allgather
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    wl = synth.workload("mlp4096", reduced=True) if len(stage_last) > 2 or reps[0] > 1 else synth.workload("mlp_small")
    p0 = synth.init_params(wl.layers)
    data = synth.make_data(wl, 5)
    plan = pd.Plan.manual(stage_last, reps)
    P = Pipeline(plan, wl.layers, p0, dtype=dtype, lr=wl.lr, minibatch=wl.batch, record_trace=1,
                 local=lambda w: w == rank, allgather=torch_allgather())
    P.set_data(*data, 5)
    dist.barrier()
    for _ in range(runs):
        P.run(M)  # flag words are monotonic across runs: the second run waits on its own messages
    s = [s for s, (a, b, r, g) in enumerate(plan.stages) if g <= rank < g + r][0]
    first, last = plan.stages[s][0], plan.stages[s][1]
    params = {l: pd.pd_get_params(P.ctx, l, synth.param_count(wl.layers[l])) for l in range(first, last + 1)}
    res = {"trace": [t[:8] for t in P.trace()], "vmap": P.version_map(M), "params": params, "stage": s}
    dist.barrier()
    P.close()
    with open(os.path.join(out_dir, f"r{rank}.pkl"), "wb") as f:
        pickle.dump(res, f)
    dist.destroy_process_group()


@pytest.mark.parametrize("stage_last,reps,M,runs", [([1, 2], [1, 1], 8, 1), ([3, 7, 11, 15], [1, 1, 1, 1], 12, 1),
                                                    ([7, 15], [2, 1], 8, 1),
                                                    # several pd_runs: replica rounds and the
                                                    # activation / gradient links continue from
                                                    # the previous run's messages
                                                    ([7, 15], [2, 1], 6, 3), ([15], [2], 4, 3),
                                                    ([3, 7, 11, 15], [1, 1, 1, 1], 9, 2)])
def test_two_processes_one_gpu_ipc(stage_last, reps, M, runs):
    import oracle
    import synth
    import torchref
    import paper_conf_sosp_narayananhpsdgg19_b200 as pd
    world = sum(reps)
    with tempfile.TemporaryDirectory() as d:
        mp.spawn(_worker, args=(world, _free_port(), stage_last, reps, pd.PD_FP32, M, d, runs), nprocs=world,
                 join=True)
        parts = [pickle.load(open(os.path.join(d, f"r{r}.pkl"), "rb")) for r in range(world)]
    wl = synth.workload("mlp4096", reduced=True) if len(stage_last) > 2 or reps[0] > 1 else synth.workload("mlp_small")
    p0 = synth.init_params(wl.layers)
    data = synth.make_data(wl, 5)
    ref = oracle.run(wl.layers, stage_last, reps, wl.batch, M, p0, data, lr=wl.lr)
    for _ in range(runs - 1):  # each pd_run continues from the previous run's parameters
        ref = oracle.run(wl.layers, stage_last, reps, wl.batch, M, ref.params, data, lr=wl.lr)
        ref.events = None
    # versions count updates over all runs: M / R_s per stage per earlier run
    ref.version_map = ref.version_map + np.array([(runs - 1) * M // r for r in reps])[:, None]
    trace = [e for p in parts for e in p["trace"]]
    if ref.events is not None:
        assert sorted(trace) == sorted(ref.events)
    for p in parts:
        s = p["stage"]
        row = p["vmap"][s]
        mask = row >= 0
        assert np.array_equal(row[mask], ref.version_map[s][mask])
        for l, v in p["params"].items():
            assert torchref.max_rel_err([v], [ref.params[l]]) < 1e-4
