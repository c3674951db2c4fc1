#!/bin/bash
# ncu evidence of round 2 (one gpurun call; results in gpurun_out/, summarised into profiles/):
#   1. launch list of the default bench (GNMT-16, N = 1): per-kernel device time
#   2. per-stage tensor-pipe activity: every stage of the 8-stage GNMT-16 plan in solo mode
#      (pd_stage_solo) with sm__pipe_tensor_cycles_active + DRAM bytes per kernel
#   3. ncu --set full of the wavefront kernels at N = 1 (16-layer run) and of stage 5 (3 layers)
#   gpurun --timeout 3000 -- bash tools/gpu_ncu_r02.sh
set -u
mkdir -p gpurun_out
B="python bench.py --no-cpu-baseline --no-e2e"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_gnmt16.csv \
  $B --steps 1 --warmup 1 --minibatches 1 --stage-plan 0 > gpurun_out/ncu_launch.log 2>&1
MET=gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed,dram__bytes_read.sum,dram__bytes_write.sum
for s in 0 1 2 3 4 5 6 7; do
  timeout 600 ncu --metrics $MET --clock-control none --csv --log-file gpurun_out/stage${s}_ncu.csv \
    python bench.py --stage $s --solo-runs 1 > gpurun_out/stage${s}_ncu.log 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:lstm_wave_kernel -s 2 -c 2 \
  -o gpurun_out/wave_n1 --force-overwrite $B --steps 1 --warmup 1 --minibatches 1 --stage-plan 0 > gpurun_out/ncu_wave_n1.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:lstm_wave_kernel -s 2 -c 2 \
  -o gpurun_out/wave_s5 --force-overwrite python bench.py --stage 5 --solo-runs 1 > gpurun_out/ncu_wave_s5.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tc_gemm_kernel -s 6 -c 3 \
  -o gpurun_out/gemm_s7 --force-overwrite python bench.py --stage 7 --solo-runs 1 > gpurun_out/ncu_gemm_s7.log 2>&1
echo done > gpurun_out/ncu_done.txt
