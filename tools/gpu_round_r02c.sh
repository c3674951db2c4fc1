#!/bin/bash
# round 2, late session: GPU suite + smoke, every config's bench line + reference arm, ncu of
# the cluster split-K GEMM in the MLP step, MLP launch list
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
B="python bench.py --no-cpu-baseline --no-e2e --config mlp4096 --stage-plan 0"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_mlp4096.csv \
  $B --steps 1 --warmup 1 --minibatches 1 > gpurun_out/ncu_launch_mlp.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:csplit2 -s 4 -c 2 \
  -o gpurun_out/csplit2 --force-overwrite $B --steps 1 --warmup 1 --minibatches 1 > gpurun_out/ncu_csplit2.log 2>&1
ncu -i gpurun_out/csplit2.ncu-rep --page raw --csv > gpurun_out/ncu_full_csplit2.csv 2>/dev/null
echo done > gpurun_out/round_done.txt
