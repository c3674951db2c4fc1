"""GEMM micro-benchmark through the C ABI (pd_kernel_gemm), CUDA events on the launching
stream, L2 flushed between iterations; for tuning tile width / split-K on the MLP shapes.
usage: gemm_bench.py [fwd|dx|dw] BN SPLIT [M N K]"""
import os, sys
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import torch
import paper_conf_sosp_narayananhpsdgg19_b200 as pd


def bench(M, N, K, amn, bmn, epi, split_ws, iters=20):
    A = (torch.randn(K, M, device="cuda") if amn else torch.randn(M, K, device="cuda")).to(torch.bfloat16)
    B = (torch.randn(K, N, device="cuda") if bmn else torch.randn(N, K, device="cuda")).to(torch.bfloat16)
    out = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
    master = torch.randn(M, N, device="cuda")
    slot = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
    bias = torch.zeros(N, device="cuda")
    ws = torch.zeros(8 * M * N, device="cuda")  # stays zero under ZEROWS=1 (workspace_zeroed contract)
    s = torch.cuda.current_stream()
    if epi == pd.PD_EPI_STORE:
        kw = dict(bias=bias.data_ptr(), relu=1)
    else:
        kw = dict(master=master.data_ptr(), slot=slot.data_ptr(), lr=1e-3)
    if split_ws:
        kw.update(workspace=ws.data_ptr(), workspace_bytes=ws.numel() * 4,
                  workspace_zeroed=int(bool(os.environ.get("ZEROWS"))))
    f = lambda: pd.pd_kernel_gemm(pd.PD_BF16, M, N, K, A.data_ptr(), A.shape[1], B.data_ptr(), B.shape[1],
                                  out.data_ptr(), N, amn, bmn, epi, stream=s.cuda_stream, **kw)
    for _ in range(3):
        f()
    flush = torch.ones(64 * 1024 * 1024, dtype=torch.float32, device="cuda")  # 256 MB, read to flush
    ts = []
    for _ in range(iters):
        if not os.environ.get("NOFLUSH"):
            flush.sum()  # clean (read-only) L2 flush: no dirty lines left to write back
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        f()
        e1.record(s)
        e1.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    ts.sort()
    return ts[len(ts) // 2]


if __name__ == "__main__":
    kind = sys.argv[1] if len(sys.argv) > 1 else "all"
    if kind == "all":
        for (cg, bn, split) in [(1, 64, 0), (1, 256, 4), (2, 128, 0), (2, 256, 0), (2, 256, 2), (2, 256, 4), (0, 0, 0)]:
            os.environ["PD_GEMM_CG"] = str(cg)
            os.environ["PD_GEMM_BN"], os.environ["PD_GEMM_SPLIT"] = str(bn), str(split)
            if cg == 0:  # the library's own choice
                for k in ("PD_GEMM_CG", "PD_GEMM_BN", "PD_GEMM_SPLIT"):
                    os.environ.pop(k)
            t = bench(256, 4096, 4096, 0, 0, pd.PD_EPI_STORE, split > 0)
            print(("fwd", cg, bn, split, round(t, 2), "us", round(2 * 256 * 4096 ** 2 / t / 1e6, 1), "TF"), flush=True)
            t = bench(256, 4096, 4096, 0, 1, pd.PD_EPI_STORE, split > 0)
            print(("dx", cg, bn, split, round(t, 2), "us", round(2 * 256 * 4096 ** 2 / t / 1e6, 1), "TF"), flush=True)
        for (M, N, K) in [(3200, 32000, 1024), (3200, 4096, 1024), (8192, 8192, 8192)]:
            t = bench(M, N, K, 0, 0, pd.PD_EPI_STORE, False)
            print(("big", M, N, K, round(t, 2), "us", round(2 * M * N * K / t / 1e6, 1), "TF"), flush=True)
        t = bench(4096, 4096, 256, 1, 1, pd.PD_EPI_SGD, False)
        print(("dw_sgd", round(t, 2), "us", round(171966464 / t / 1e3, 1), "GB/s"))
    else:
        bn, split = int(sys.argv[2]), int(sys.argv[3])
        os.environ["PD_GEMM_BN"], os.environ["PD_GEMM_SPLIT"] = str(bn), str(split)
        M, N, K = (int(x) for x in sys.argv[4:7]) if len(sys.argv) > 6 else (256, 4096, 4096)
        amn, bmn, epi = {"fwd": (0, 0, pd.PD_EPI_STORE), "dx": (0, 1, pd.PD_EPI_STORE),
                         "dw": (1, 1, pd.PD_EPI_SGD)}[kind]
        print(kind, bn, split, bench(M, N, K, amn, bmn, epi, split > 0, iters=5))
