#!/bin/bash
mkdir -p gpurun_out
{
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -k "store_bias or mask_epilogue or fused_update" 2>&1 | grep -v "^tests.*PASSED" | tail -60
echo "--- dw sgd BN 128 vs 256"
python tools/gemm_bench.py dw 128 0 4096 4096 256; PD_UPD_BN_SGD=256 python tools/gemm_bench.py dw 128 0 4096 4096 256
B="timeout 300 python bench.py --steps 20 --no-cpu-baseline --no-e2e"
echo "--- mlp BN_SGD=128"; $B | cut -c1-170
echo "--- mlp BN_SGD=256"; PD_UPD_BN_SGD=256 $B | cut -c1-170
} > gpurun_out/exp4.log 2>&1
