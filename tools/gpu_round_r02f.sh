#!/bin/bash
# round 2, final: GPU suite + smoke, every config's bench line + reference arm, ncu launch lists of
# the default (GNMT-16) and VGG-16 steps
set -u
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu,power.limit --format=csv > gpurun_out/gpu.txt 2>&1
timeout 1800 python -m pytest tests -m gpu -q -rf --durations=15 > gpurun_out/pytest_gpu.log 2>&1
echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke exit $?" >> gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench_gnmt16.json 2> gpurun_out/bench_gnmt16.err
for c in mlp4096 gnmt8 vgg16; do
  timeout 600 python bench.py --config $c --no-cpu-baseline --stage-plan 0 > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err
done
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
for c in gnmt16 vgg16; do
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$c.csv \
    python bench.py --config $c --no-cpu-baseline --no-e2e --stage-plan 0 --steps 1 --warmup 1 --minibatches 1 > /dev/null 2>&1
done
echo done > gpurun_out/round_done.txt
