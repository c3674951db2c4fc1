"""N > 1 host path on CPU: two processes over torch.distributed (gloo, world size 2), as
`bench.py --gpus 2` launches them under torchrun, minus the GPU.

Covers what every rank computes on its own and must agree on without a data-path exchange
(SURVEY §8(e)): the plan (pd_plan is deterministic, L855-985), the worker -> rank placement (R18),
the rank -> stage map the bench's per-rank roofline uses, the in-flight counts (k_s, L1021), the
IPC-blob all-gather plumbing of session.Pipeline (rank order, every blob delivered once), the
max-over-ranks timing reduction, and that the device path still fails loudly (no CPU fallback)
on every rank."""
import os
import pickle
import socket
import sys
import tempfile

import pytest
import torch
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rank_main(rank, world, port, out_dir):
    sys.path.insert(0, ROOT)
    import torch.distributed as dist
    import bench
    import synth
    import paper_conf_sosp_narayananhpsdgg19_b200 as pd
    from paper_conf_sosp_narayananhpsdgg19_b200.session import stage_of_rank, torch_allgather, workers_of

    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    peaks = {"hbm_gbs": 6500.0, "bf16_tflops": 1600.0, "bf16_tflops_sustained": 1380.0, "source": "test"}
    res = {"rank": rank, "plans": {}}
    for cfg, mode in (("gnmt8", "pipeline"), ("gnmt16", "pipeline"), ("mlp4096", "pipeline"), ("vgg16", "pipeline"),
                      ("mlp4096", "dp")):
        wl = synth.workload(cfg)
        plan = bench.choose_plan(cfg, mode, world, wl.layers, wl.batch, peaks)
        me = [w for w in workers_of(plan) if w[3] == rank]
        s = stage_of_rank(plan, rank)
        res["plans"][(cfg, mode)] = (plan.stages, plan.noam, s, me, pd.pd_inflight(plan))
    # IPC-blob exchange plumbing (what Pipeline does with pd_export_worker blobs)
    ag = torch_allgather()
    res["gathered"] = ag([f"blob-r{rank}-{k}".encode() for k in range(rank + 1)])
    # max over ranks of a per-rank step time (bench.py allmax, gloo here)
    t = torch.tensor([1.0 + rank], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    res["max"] = float(t.item())
    # the device path fails loudly on every rank (no CPU fallback)
    wl = synth.workload("mlp_small")
    plan = pd.Plan.manual([1, 2], [1, 1])
    ctx = pd.pd_create(plan, wl.layers, pd.PD_FP32, minibatch=wl.batch)
    p0 = synth.init_params(wl.layers)
    s = stage_of_rank(plan, rank)
    try:
        first, last = plan.stages[s][0], plan.stages[s][1]
        pd.pd_stage_init(ctx, s, 0, 0, [p0[l] for l in range(first, last + 1)])
        res["stage_init"] = "ok"
    except pd.PDError as e:
        res["stage_init"] = e.status
    pd.pd_destroy(ctx)
    dist.barrier()
    dist.destroy_process_group()
    with open(os.path.join(out_dir, f"r{rank}.pkl"), "wb") as f:
        pickle.dump(res, f)


@pytest.mark.skipif(torch.cuda.is_available(), reason="CPU-only host-path test (the GPU box runs test_gpu_multiproc)")
def test_two_ranks_agree_on_plan_placement_and_exchange():
    import paper_conf_sosp_narayananhpsdgg19_b200 as pd
    world = 2
    with tempfile.TemporaryDirectory() as d:
        mp.spawn(_rank_main, args=(world, _free_port(), d), nprocs=world, join=True)
        parts = [pickle.load(open(os.path.join(d, f"r{r}.pkl"), "rb")) for r in range(world)]
    r0, r1 = parts
    for key in r0["plans"]:
        st0, noam0, s0, me0, k0 = r0["plans"][key]
        st1, noam1, s1, me1, k1 = r1["plans"][key]
        # same plan and in-flight counts on both ranks, computed independently
        assert st0 == st1 and noam0 == noam1 and k0 == k1, key
        # every GPU used exactly once (sum R_s = W), one worker per rank, consecutive placement
        assert sum(s[2] for s in st0) == world
        assert len(me0) == 1 and len(me1) == 1 and me0[0][3] == 0 and me1[0][3] == 1
        assert me0[0][1] == s0 and me1[0][1] == s1
    # straight 2-stage pipelines for the pd_plan configs: rank 0 -> stage 0, rank 1 -> stage 1,
    # NOAM = 2 and k = (2, 1) (L1021)
    for key in (("gnmt8", "pipeline"), ("gnmt16", "pipeline"), ("mlp4096", "pipeline")):
        st, noam, s, me, k = r0["plans"][key]
        assert len(st) == 2 and [x[2] for x in st] == [1, 1] and noam == 2 and list(k) == [2, 1], key
        assert r1["plans"][key][2] == 1
    # VGG at N = 2 is the (N-1)-1 = 1-1 plan; pure DP is one stage x 2 replicas (NOAM = 1)
    st, noam, s, me, k = r0["plans"][("vgg16", "pipeline")]
    assert [x[2] for x in st] == [1, 1] and noam == 2
    st, noam, s, me, k = r0["plans"][("mlp4096", "dp")]
    assert len(st) == 1 and st[0][2] == 2 and noam == 1 and me == [(0, 0, 0, 0)]
    assert r1["plans"][("mlp4096", "dp")][3] == [(1, 0, 1, 1)]
    # all-gather: rank order, every rank's blobs exactly once, identical on both ranks
    want = [[b"blob-r0-0"], [b"blob-r1-0", b"blob-r1-1"]]
    assert r0["gathered"] == want and r1["gathered"] == want
    assert r0["max"] == r1["max"] == 2.0
    assert r0["stage_init"] in (pd.PD_ECUDA, pd.PD_EUNSUPPORTED)
    assert r1["stage_init"] in (pd.PD_ECUDA, pd.PD_EUNSUPPORTED)
