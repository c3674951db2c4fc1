#!/bin/bash
mkdir -p gpurun_out
{
P='import sys,json; d=json.loads(sys.stdin.read()); print(round(d["value"]), round(d["step_share"]["fwd_gemm"],3), round(d["step_share"]["dx_gemm"],3))'
B="timeout 300 python bench.py --steps 20 --no-cpu-baseline --no-e2e"
echo "--- mlp default"; $B | python -c "$P"
for cs in 2 3 4; do for ep in 1 3; do
  echo "--- mlp CSPLIT=$cs EPI=$ep"; PD_GEMM_CSPLIT=$cs PD_GEMM_CSPLIT_EPI=$ep $B | python -c "$P"
done; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_vgg16.csv \
    python bench.py --config vgg16 --steps 1 --warmup 1 --minibatches 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
python tools/launches.py gpurun_out/launches_vgg16.csv | tail -25
} > gpurun_out/exp12.log 2>&1
