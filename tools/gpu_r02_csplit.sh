# cluster split-K bring-up: kernel parity, isolated / chained timings, phase probe
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -rf -x -k "cluster_splitk or store_bias or mask_epilogue or split_k_reduction" > gpurun_out/pytest_csplit.log 2>&1; echo "exit $?" >> gpurun_out/pytest_csplit.log
timeout 300 python tools/csplit_bench.py > gpurun_out/csplit_bench.log 2>&1
for m in 2 1; do PD_GEMM_CSPLIT=$m timeout 300 python tools/gemm_probe.py 256 4096 4096 >> gpurun_out/csplit_probe.log 2>&1; done
for cs in 2 0; do PD_GEMM_CSPLIT=$cs timeout 600 python bench.py --config mlp4096 --no-cpu-baseline --stage-plan 0 > gpurun_out/bench_mlp4096_cs$cs.json 2> gpurun_out/bench_mlp4096_cs$cs.err; done
