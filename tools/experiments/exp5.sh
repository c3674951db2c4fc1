#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/wave_probe.txt
PD_WAVE_PROBE=gpurun_out/wave_probe.txt timeout 300 python bench.py --config gnmt8 --steps 1 --warmup 1 --minibatches 1 --no-cpu-baseline --no-e2e > gpurun_out/exp5.log 2>&1
python tools/wave_probe.py gpurun_out/wave_probe.txt >> gpurun_out/exp5.log 2>&1
