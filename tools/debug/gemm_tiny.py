import os, sys
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import torch
import paper_conf_sosp_narayananhpsdgg19_b200 as pd
from gemm_bench import bench
os.environ["NOFLUSH"] = "1"
for cg in ("1", "2"):
    os.environ["PD_GEMM_CG"] = cg
    for (M, N, K) in [(128, 128, 64), (256, 256, 64), (256, 256, 1024), (256, 4096, 64), (256, 4096, 1024)]:
        t = bench(M, N, K, 0, 0, pd.PD_EPI_STORE, False)
        print("cg", cg, (M, N, K), round(t, 2), "us", flush=True)
s = torch.cuda.current_stream()
x = torch.zeros(16, device="cuda")
ts = []
for _ in range(20):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s); x.add_(1); e1.record(s); e1.synchronize(); ts.append(e0.elapsed_time(e1) * 1e3)
print("tiny torch kernel", sorted(ts)[10], "us")
