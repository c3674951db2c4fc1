#!/bin/bash
# L2-prefetch experiment: isolated M=256 GEMMs (L2 flushed vs warm), probe, and the MLP step with
# PD_L2_PF = 0..3.  gpurun -- bash tools/experiments/exp_pf.sh
mkdir -p gpurun_out
{
python tools/gemm_bench.py all
echo "--- NOFLUSH"
NOFLUSH=1 python tools/gemm_bench.py all
echo "--- probe"
python tools/gemm_probe.py
for pf in 0 1 2 3; do
  echo "--- PD_L2_PF=$pf"
  PD_L2_PF=$pf timeout 300 python bench.py --steps 20 --no-cpu-baseline --no-e2e
done
} > gpurun_out/exp_pf.log 2>&1
