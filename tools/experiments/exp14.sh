#!/bin/bash
mkdir -p gpurun_out
{
timeout 900 python -m pytest tests/test_gpu_kernels.py -x -q -k "split_k_reduction_modes" 2>&1 | tail -2
timeout 900 python -m pytest tests/test_gpu_lstm_rec.py -x -q -k "wave" 2>&1 | tail -2
P='import sys,json; d=json.loads(sys.stdin.read()); print(round(d["value"]), round(d["step_share"]["fwd_gemm"],3), round(d["step_share"]["dx_gemm"],3))'
B="timeout 300 python bench.py --steps 20 --no-cpu-baseline --no-e2e"
for m in 0 2 1 0 2; do echo "--- mlp PD_SPLIT_INKERNEL=$m"; PD_SPLIT_INKERNEL=$m $B | python -c "$P"; done
rm -f gpurun_out/wave_probe.txt
PD_WAVE_PROBE=gpurun_out/wave_probe.txt timeout 300 python bench.py --config gnmt8 --steps 1 --warmup 1 --minibatches 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
python tools/wave_probe.py gpurun_out/wave_probe.txt | tail -12
for cfg in gnmt8; do echo "--- $cfg"; $B --config $cfg | python -c "$P"; done
} > gpurun_out/exp14.log 2>&1
