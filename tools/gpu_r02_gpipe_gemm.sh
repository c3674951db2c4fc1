mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_gpipe.py -q -rf -x > gpurun_out/pytest_gpipe.log 2>&1; echo "exit $?" >> gpurun_out/pytest_gpipe.log
timeout 300 python tools/cublas_ref.py > gpurun_out/cublas_ref.log 2>&1
timeout 300 python tools/gemm_probe.py > gpurun_out/gemm_probe.log 2>&1
timeout 300 python tools/gemm_bench.py all > gpurun_out/gemm_bench.log 2>&1
nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a tools/tma_bw.cu -o /tmp/tma_bw -lcuda && timeout 300 /tmp/tma_bw > gpurun_out/tma_bw.log 2>&1
