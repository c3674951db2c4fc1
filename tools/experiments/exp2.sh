#!/bin/bash
# A/B of the split-K reduce-add workspace, the split dW path and the 2-CTA tile-width choice
mkdir -p gpurun_out
{
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_lstm_rec.py -x -q -k "store_bias or mask_epilogue or split_weight" 2>&1 | tail -3
echo "--- gemm fwd/dx per-split partials vs zeroed workspace"
python tools/gemm_bench.py fwd 256 4; ZEROWS=1 python tools/gemm_bench.py fwd 256 4
python tools/gemm_bench.py dx 256 4; ZEROWS=1 python tools/gemm_bench.py dx 256 4
B="timeout 300 python bench.py --steps 20 --no-cpu-baseline --no-e2e"
echo "--- mlp atomic (default)"; $B | cut -c1-200
echo "--- mlp PD_SPLIT_ATOMIC=0"; PD_SPLIT_ATOMIC=0 $B | cut -c1-200
for cfg in gnmt8 vgg16; do
  echo "--- $cfg default"; $B --config $cfg | cut -c1-200
  echo "--- $cfg BNSEL=0"; PD_GEMM_BNSEL=0 $B --config $cfg | cut -c1-200
done
for k in 512 1024 2048; do echo "--- gnmt8 DW_SPLIT_K=$k"; PD_DW_SPLIT_K=$k $B --config gnmt8 | cut -c1-200; done
echo "--- vgg16 DW_SPLIT_K=1024"; PD_DW_SPLIT_K=1024 $B --config vgg16 | cut -c1-200
} > gpurun_out/exp2.log 2>&1
