#!/bin/bash
mkdir -p gpurun_out
{
timeout 900 python -m pytest tests/test_gpu_lstm_rec.py tests/test_gpu_pipeline.py -x -q -k "gnmt or GNMT or lstm or wave or split" 2>&1 | tail -2
rm -f gpurun_out/wave_probe.txt
PD_WAVE_PROBE=gpurun_out/wave_probe.txt timeout 300 python bench.py --config gnmt8 --steps 1 --warmup 1 --minibatches 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
python tools/wave_probe.py gpurun_out/wave_probe.txt
B="timeout 400 python bench.py --steps 20 --no-cpu-baseline --no-e2e"
for cfg in gnmt8; do echo "--- $cfg"; $B --config $cfg | cut -c1-200; done
} > gpurun_out/exp10.log 2>&1
