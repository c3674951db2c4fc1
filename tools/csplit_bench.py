"""Cluster split-K vs workspace split-K for the MLP-4096 small-M GEMMs (tools only): CUDA-event
medians per launch, with and without an L2 flush before each launch, and back-to-back chains of
16 launches (the forward of a 16-layer stage).  usage: csplit_bench.py"""
import os
import sys
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import torch
import paper_conf_sosp_narayananhpsdgg19_b200 as pd

M, N, K = 256, 4096, 4096


def main():
    X = [torch.randn(M, K, device="cuda").bfloat16() for _ in range(17)]
    Ws = [torch.randn(N, K, device="cuda").bfloat16() for _ in range(16)]
    bias = torch.zeros(N, device="cuda")
    mask = torch.ones(M, N, device="cuda").bfloat16()
    ws = torch.zeros(8 * M * N, device="cuda")
    flush = torch.ones(64 * 1024 * 1024, device="cuda")
    s = torch.cuda.current_stream()

    def gemm(i, dx=False):
        kw = dict(workspace=ws.data_ptr(), workspace_bytes=ws.numel() * 4, stream=s.cuda_stream)
        if dx:
            pd.pd_kernel_gemm(pd.PD_BF16, M, N, K, X[i].data_ptr(), K, Ws[i].data_ptr(), N, X[i + 1].data_ptr(), N,
                              0, 1, pd.PD_EPI_MASK, mask=mask.data_ptr(), ldm=N, **kw)
        else:
            pd.pd_kernel_gemm(pd.PD_BF16, M, N, K, X[i].data_ptr(), K, Ws[i].data_ptr(), K, X[i + 1].data_ptr(), N,
                              0, 0, pd.PD_EPI_STORE, bias=bias.data_ptr(), relu=1, **kw)

    def timed(f, reps=30, fl=False):
        ts = []
        for _ in range(reps):
            if fl:
                flush.sum()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            f()
            b.record(s)
            b.synchronize()
            ts.append(a.elapsed_time(b) * 1e3)
        ts.sort()
        return ts[len(ts) // 2]

    for cs in ("2", "1", "0"):
        os.environ["PD_GEMM_CSPLIT"] = cs
        for dx in (False, True):
            gemm(0, dx)
            t_flush = timed(lambda: gemm(0, dx), fl=True)
            t_warm = timed(lambda: gemm(0, dx))
            t_chain = timed(lambda: [gemm(i, dx) for i in range(16)], reps=10, fl=True) / 16
            print(f"csplit={cs} {'dX ' if dx else 'fwd'}: flushed {t_flush:6.2f} us  warm {t_warm:6.2f} us  "
                  f"16-chain {t_chain:6.2f} us/layer", flush=True)


if __name__ == "__main__":
    main()
