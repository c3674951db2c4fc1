import os, sys
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import paper_conf_sosp_narayananhpsdgg19_b200 as pd
from gemm_bench import bench
for (M, N, K) in [(256, 4096, 4096), (512, 4096, 4096), (1024, 4096, 4096), (2048, 4096, 4096), (4096, 4096, 4096),
                  (256, 16384, 4096), (256, 4096, 16384), (1024, 1024, 4096), (4096, 4096, 256)]:
    t = bench(M, N, K, 0, 0, pd.PD_EPI_STORE, True)
    print((M, N, K), round(t, 2), "us", round(2 * M * N * K / t / 1e6, 1), "TF", flush=True)
