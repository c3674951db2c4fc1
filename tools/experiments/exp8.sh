#!/bin/bash
mkdir -p gpurun_out
{
timeout 600 python -m pytest tests/test_gpu_kernels.py -x -q -k "fused_update" 2>&1 | tail -3
echo "--- dw sgd resident-B vs strided"
python tools/gemm_bench.py dw 128 0 4096 4096 256; PD_UPD_RESB=0 python tools/gemm_bench.py dw 128 0 4096 4096 256
B="timeout 300 python bench.py --steps 20 --no-cpu-baseline --no-e2e"
echo "--- mlp RESB=1"; $B | cut -c1-170
echo "--- mlp RESB=0"; PD_UPD_RESB=0 $B | cut -c1-170
echo "--- mlp RESB=1 again"; $B | python -c "import sys,json; d=json.loads(sys.stdin.read()); print(d['value'], d['roofline']['avg_launch_us'], d['roofline']['frac'])"
} > gpurun_out/exp8.log 2>&1
