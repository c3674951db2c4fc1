import os, sys
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import paper_conf_sosp_narayananhpsdgg19_b200 as pd
from gemm_bench import bench
for split in ("0", "1"):
    os.environ["PD_GEMM_SPLIT"] = split
    for (M, N, K) in [(256, 4096, 4096), (4096, 256, 4096), (512, 2048, 4096), (2048, 512, 4096)]:
        t = bench(M, N, K, 0, 0, pd.PD_EPI_STORE, True)
        print("split", split, (M, N, K), round(t, 2), "us", flush=True)
