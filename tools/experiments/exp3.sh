#!/bin/bash
mkdir -p gpurun_out
{
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
B="timeout 400 python bench.py --steps 20 --no-cpu-baseline --no-e2e"
for cfg in mlp4096 gnmt8 gnmt16 vgg16; do echo "--- $cfg"; $B --config $cfg; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_gnmt8.csv \
    python bench.py --config gnmt8 --steps 1 --warmup 1 --minibatches 2 --no-cpu-baseline --no-e2e > /dev/null 2>&1
} > gpurun_out/exp3.log 2>&1
