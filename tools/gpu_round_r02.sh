#!/bin/bash
# One gpurun call of round 2: GPU tests, smoke, bench lines of every config + the reference
# arm, the per-stage projection of GNMT-8 / GNMT-16 plans (Fig. 15 beyond one GPU).
#   gpurun --timeout 3300 -- bash tools/gpu_round_r02.sh [tests|bench|sweep|all]
set -u
what=${1:-all}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu,power.limit --format=csv > gpurun_out/gpu.txt 2>&1
if [[ $what == all || $what == tests ]]; then
  timeout 1800 python -m pytest tests -m gpu -q -rf --durations=15 > gpurun_out/pytest_gpu.log 2>&1
  echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
  timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1
  echo "smoke exit $?" >> gpurun_out/smoke.log
fi
if [[ $what == all || $what == bench ]]; then
  timeout 900 python bench.py > gpurun_out/bench_gnmt16.json 2> gpurun_out/bench_gnmt16.err
  for c in gnmt8 mlp4096 vgg16; do
    timeout 600 python bench.py --config $c --no-cpu-baseline --stage-plan 0 > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err
  done
  timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
fi
if [[ $what == all || $what == sweep ]]; then
  for c in gnmt8 gnmt16; do
    timeout 1200 python tools/plan_sweep.py --config $c --gpus 2 4 8 --real-stages --json gpurun_out/plan_sweep_$c.json \
      > gpurun_out/plan_sweep_$c.log 2>&1
  done
fi
echo done > gpurun_out/round_done.txt
