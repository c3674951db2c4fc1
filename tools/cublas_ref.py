"""Library reference point for the small-M GEMMs (tools only, never on the product path):
cuBLAS through torch.matmul on the MLP-4096 forward / dX shapes, CUDA events, L2 flushed
(read-only sweep) before every launch, weights cold like in the pipeline.
usage: cublas_ref.py"""
import torch


def t_us(f, iters=30):
    flush = torch.ones(64 * 1024 * 1024, dtype=torch.float32, device="cuda")
    for _ in range(3):
        f()
    s = torch.cuda.current_stream()
    ts = []
    for _ in range(iters):
        flush.sum()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        f()
        b.record(s)
        b.synchronize()
        ts.append(a.elapsed_time(b) * 1e3)
    ts.sort()
    return ts[len(ts) // 2]


if __name__ == "__main__":
    M, N, K = 256, 4096, 4096
    X = torch.randn(M, K, device="cuda").bfloat16()
    W = torch.randn(N, K, device="cuda").bfloat16()
    G = torch.randn(M, N, device="cuda").bfloat16()
    flop = 2 * M * N * K
    for name, f in (("fwd X W^T", lambda: X @ W.t()), ("dX G W", lambda: G @ W),
                    ("fwd+bias+relu", lambda: torch.relu(torch.nn.functional.linear(X, W)))):
        t = t_us(f)
        print(f"cublas {name:14s} {t:7.2f} us  {flop / t / 1e6:7.1f} TF/s", flush=True)
