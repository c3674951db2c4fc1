#!/bin/bash
# One gpurun call: GPU tests, smoke, bench lines for every config, launch list, ncu full of the
# dominant kernel. Results land in gpurun_out/ (merged back by gpurun).
#   gpurun --timeout 3000 -- bash tools/gpu_round.sh [tests|bench|ncu|all]
set -u
what=${1:-all}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv > gpurun_out/gpu.txt 2>&1
if [[ $what == all || $what == tests ]]; then
  timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1
  echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
  timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1
  echo "smoke exit $?" >> gpurun_out/smoke.log
fi
if [[ $what == all || $what == bench ]]; then
  timeout 400 python bench.py > gpurun_out/bench_mlp4096.json 2> gpurun_out/bench_mlp4096.err
  for c in gnmt8 gnmt16 vgg16; do
    timeout 500 python bench.py --config $c --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err
  done
  timeout 400 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
fi
if [[ $what == all || $what == ncu ]]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_mlp4096.csv \
    python bench.py --steps 1 --warmup 1 --minibatches 2 --no-cpu-baseline --no-e2e > /dev/null 2>&1
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:tc_gemm_update -s 8 -c 1 \
    -o gpurun_out/dw_update --force-overwrite \
    python bench.py --steps 1 --warmup 1 --minibatches 2 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full.log 2>&1
fi
if [[ $what == all || $what == ncu || $what == ncu_gnmt ]]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_gnmt8.csv \
    python bench.py --config gnmt8 --steps 1 --warmup 1 --minibatches 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:lstm_wave_kernel -c 2 \
    -o gpurun_out/lstm_wave --force-overwrite \
    python bench.py --config gnmt8 --steps 1 --warmup 1 --minibatches 1 --no-cpu-baseline --no-e2e > gpurun_out/ncu_wave.log 2>&1
fi
echo done > gpurun_out/round_done.txt
