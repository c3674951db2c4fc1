# PDL for the forward GEMM chain: parity (kernel + pipeline tests, GPipe) then MLP bench with / without
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_gpipe.py tests/test_gpu_pipeline.py tests/test_gpu_stash_bf16.py -q -rf -x > gpurun_out/pytest_pdl.log 2>&1; echo "exit $?" >> gpurun_out/pytest_pdl.log
for pdl in 1 0; do PD_GEMM_PDL=$pdl timeout 600 python bench.py --config mlp4096 --no-cpu-baseline --stage-plan 0 > gpurun_out/bench_mlp4096_pdl$pdl.json 2> gpurun_out/bench_mlp4096_pdl$pdl.err; done
