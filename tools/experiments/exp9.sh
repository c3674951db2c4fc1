#!/bin/bash
mkdir -p gpurun_out
{
PD_UPD_DEEP=1 timeout 600 python -m pytest tests/test_gpu_kernels.py -x -q -k "fused_update" 2>&1 | tail -2
echo "--- dw sgd default vs DEEP"
python tools/gemm_bench.py dw 128 0 4096 4096 256; PD_UPD_DEEP=1 python tools/gemm_bench.py dw 128 0 4096 4096 256
B="timeout 300 python bench.py --steps 20 --no-cpu-baseline --no-e2e"
echo "--- mlp default"; $B | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['roofline']['avg_launch_us'], d['roofline']['frac'])"
echo "--- mlp DEEP"; PD_UPD_DEEP=1 $B | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['roofline']['avg_launch_us'], d['roofline']['frac'])"
} > gpurun_out/exp9.log 2>&1
