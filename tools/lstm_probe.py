"""Time the persistent LSTM recurrence kernels alone (CUDA events) and break a step into
phases from the in-kernel %globaltimer stamps (pd_kernel_lstm_rec probe buffer).

    python tools/lstm_probe.py [--H 1024] [--B 64] [--T 50]

Phases (per CTA, thread 0's view): 0 step start, 1 dependencies met + TMA issued, 2 MMAs
done, 3 partial staged + cluster barrier, 4 DSMEM reduction read, 5 cell + stores + publish;
stamps 6/7 of step 0 = kernel entry / prologue (weights into shared memory) done."""
import argparse
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sosp_narayananhpsdgg19_b200 as pd  # noqa: E402


def summarize(name, pr, T):
    pr = pr.astype(np.int64)
    ent, pro = pr[:, 0, 6], pr[:, 0, 7]
    t0 = ent.min()
    print(f"{name}: prologue median {np.median(pro - ent) / 1e3:.1f} us (max {np.max(pro - t0) / 1e3:.1f} us "
          f"after the first CTA entered)")
    s = pr[:, 1:, :6]  # steps >= 1 (they run the MMA path)
    d = np.diff(s, axis=2) / 1e3
    names = ["deps+TMA issue", "TMA+MMA", "stage+cluster sync", "DSMEM reduce", "cell+publish"]
    for i, n in enumerate(names):
        print(f"   {n:20s} median {np.median(d[:, :, i]):6.2f} us  p90 {np.percentile(d[:, :, i], 90):6.2f}")
    per = np.diff(pr[:, :, 0], axis=1) / 1e3
    print(f"   step period median {np.median(per):.2f} us; whole recurrence "
          f"{(pr[:, -1, 5].max() - t0) / 1e3:.1f} us")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--H", type=int, default=1024)
    ap.add_argument("--B", type=int, default=64)
    ap.add_argument("--T", type=int, default=50)
    ap.add_argument("--reps", type=int, default=20)
    a = ap.parse_args()
    H, B, T = a.H, a.B, a.T
    dev = torch.device("cuda")
    g = torch.Generator(device="cpu").manual_seed(0)
    k = 1.0 / np.sqrt(H)
    W = ((torch.rand(4 * H, H, generator=g) * 2 - 1) * k).to(torch.bfloat16).to(dev)
    gx = (torch.randn(T, B, 4 * H, generator=g) * 0.5).to(dev)
    bih = ((torch.rand(4 * H, generator=g) * 2 - 1) * k).to(dev)
    bhh = ((torch.rand(4 * H, generator=g) * 2 - 1) * k).to(dev)
    gates = torch.empty(T, B, 4 * H, device=dev)
    c = torch.empty(T, B, H, device=dev)
    h = torch.empty(T, B, H, device=dev, dtype=torch.bfloat16)
    dy = (torch.randn(T, B, H, generator=g) * 0.1).to(torch.bfloat16).to(dev)
    da = torch.empty(T, B, 4 * H, device=dev, dtype=torch.bfloat16)
    cnt = torch.zeros(1024, device=dev, dtype=torch.int32)
    grid = {0: H // 8, 1: H // 16}
    st = torch.cuda.current_stream().cuda_stream

    def call(direction, probe=None):
        pd.pd_kernel_lstm_rec(direction, T, B, H, W.data_ptr(), gates.data_ptr(), c.data_ptr(), cnt.data_ptr(),
                              gx=gx.data_ptr(), b_ih=bih.data_ptr(), b_hh=bhh.data_ptr(), h=h.data_ptr(),
                              dy=dy.data_ptr(), da=da.data_ptr(), probe=probe, stream=st)

    # bring the SM clock up before timing (an idle B200 sits at ~120 MHz) with the kernel
    # itself: a matmul warm-up hits the power cap and leaves the clock low
    for _ in range(400):
        call(0)
    torch.cuda.synchronize()
    import subprocess
    print(subprocess.run(["nvidia-smi", "--query-gpu=clocks.sm,clocks.max.sm", "--format=csv,noheader"],
                         capture_output=True, text=True).stdout.strip())
    for direction, name in ((0, "forward"), (1, "backward")):
        for _ in range(3):
            call(direction)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(a.reps):
            call(direction)
        e1.record()
        torch.cuda.synchronize()
        us = e0.elapsed_time(e1) * 1e3 / a.reps
        flops = 2.0 * B * 4 * H * H * (T - 1)
        print(f"{name}: {us:.1f} us per launch ({us / T:.2f} us/step, recurrent GEMM {flops / us / 1e6:.1f} TFLOP/s)")
        pr = torch.zeros(grid[direction], T, 8, dtype=torch.int64, device=dev)
        call(direction, probe=pr.data_ptr())
        torch.cuda.synchronize()
        summarize(name, pr.cpu().numpy(), T)
    print("h finite:", bool(torch.isfinite(h.float()).all()), "da finite:", bool(torch.isfinite(da.float()).all()))


if __name__ == "__main__":
    main()
