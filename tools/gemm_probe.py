"""Per-CTA phase timeline of the tcgen05 GEMM (PD_GEMM_PROBE stamps, %globaltimer ns):
entry, setup done, first TMA issued, 1st stage full, 2nd stage full, last MMA issued,
accumulator ready, epilogue done.  usage: gemm_probe.py  (prints medians / maxima per config)"""
import os
import sys
import tempfile

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
path = os.path.join(tempfile.gettempdir(), "pd_probe.txt")
os.environ["PD_GEMM_PROBE"] = path
import numpy as np  # noqa: E402
import torch  # noqa: E402
import paper_conf_sosp_narayananhpsdgg19_b200 as pd  # noqa: E402

NAMES = ["entry", "setup", "tma0", "full0", "full1", "lastmma", "accrdy", "ld0", "chunk0", "chunk1", "loopend",
         "epidone"]


def run(M, N, K, env, amn=0, bmn=0, epi=pd.PD_EPI_STORE, reps=3):
    for k in ("PD_GEMM_CG", "PD_GEMM_BN", "PD_GEMM_SPLIT"):
        os.environ.pop(k, None)
    os.environ.update({k: str(v) for k, v in env.items()})
    A = (torch.randn(K, M, device="cuda") if amn else torch.randn(M, K, device="cuda")).to(torch.bfloat16)
    B = (torch.randn(K, N, device="cuda") if bmn else torch.randn(N, K, device="cuda")).to(torch.bfloat16)
    out = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
    bias = torch.zeros(N, device="cuda")
    ws = torch.empty(8 * M * N, device="cuda")
    flush = torch.ones(64 * 1024 * 1024, dtype=torch.float32, device="cuda")
    if os.path.exists(path):
        os.remove(path)
    for _ in range(reps):
        flush.sum()
        torch.cuda.synchronize()
        pd.pd_kernel_gemm(pd.PD_BF16, M, N, K, A.data_ptr(), A.shape[1], B.data_ptr(), B.shape[1], out.data_ptr(),
                          N, amn, bmn, epi, bias=bias.data_ptr(), relu=1, workspace=ws.data_ptr(),
                          workspace_bytes=ws.numel() * 4, stream=torch.cuda.current_stream().cuda_stream)
        torch.cuda.synchronize()
    lines = open(path).read().strip().split("\n")
    last = lines[-1]
    head, *ctas = last.split("|")
    arr = np.array([[int(x) for x in c.split()] for c in ctas], dtype=np.float64) / 1000.0  # us
    arr[arr < 0] = np.nan
    med = np.nanmedian(arr, axis=0)
    mx = np.nanmax(arr, axis=0)
    print(f"{head.strip()} {env}")
    print("   median us: " + " ".join(f"{n}={v:.2f}" for n, v in zip(NAMES, med)))
    if os.environ.get("PROBE_ALL"):
        for row in arr:
            print("      " + " ".join(f"{v:.2f}" for v in row))
    print("   max    us: " + " ".join(f"{n}={v:.2f}" for n, v in zip(NAMES, mx)), flush=True)


if __name__ == "__main__":
    if len(sys.argv) > 1:
        M, N, K = (int(x) for x in sys.argv[1:4])
        env = dict(kv.split("=") for kv in sys.argv[4:])
        run(M, N, K, env)
        sys.exit(0)
    run(256, 4096, 4096, {})
    run(256, 4096, 4096, {"PD_GEMM_SPLIT": 1})
    run(256, 4096, 4096, {"PD_GEMM_SPLIT": 2})
    run(256, 4096, 4096, {"PD_GEMM_SPLIT": 8})
    run(256, 4096, 4096, {"PD_GEMM_CG": 1, "PD_GEMM_BN": 256, "PD_GEMM_SPLIT": 4})
    run(256, 4096, 4096, {"PD_GEMM_CG": 1, "PD_GEMM_BN": 128, "PD_GEMM_SPLIT": 2})
    run(256, 4096, 4096, {}, bmn=1)
    run(256, 4096, 1024, {"PD_GEMM_SPLIT": 1})
    run(8192, 8192, 8192, {})
    run(3200, 4096, 1024, {})
