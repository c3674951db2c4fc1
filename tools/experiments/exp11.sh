#!/bin/bash
mkdir -p gpurun_out
{
echo "--- tests with PD_PDL=1"
PD_PDL=1 timeout 900 python -m pytest tests/test_gpu_pipeline.py tests/test_gpu_kernels.py -x -q 2>&1 | tail -2
P='import sys,json; d=json.loads(sys.stdin.read()); print(round(d["value"]), d["step_share"]["fwd_gemm"], d["step_share"]["dx_gemm"])'
B="timeout 300 python bench.py --steps 20 --no-cpu-baseline --no-e2e"
for pdl in 0 1 0 1; do echo "--- mlp PD_PDL=$pdl"; PD_PDL=$pdl $B | python -c "$P"; done
for mb in 0 32 48 64 80; do echo "--- gnmt8 PD_WAVE_L2_MB=$mb"; PD_WAVE_L2_MB=$mb $B --config gnmt8 | python -c "$P"; done
rm -f gpurun_out/wave_probe.txt
PD_WAVE_L2_MB=48 PD_WAVE_PROBE=gpurun_out/wave_probe.txt timeout 300 python bench.py --config gnmt8 --steps 1 --warmup 1 --minibatches 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
python tools/wave_probe.py gpurun_out/wave_probe.txt
} > gpurun_out/exp11.log 2>&1
