# GNMT-16 N = 1: how many MB of wavefront weights to keep L2-resident (evict_last)
mkdir -p gpurun_out
for mb in 64 32 96 80 48; do
  PD_WAVE_L2_MB=$mb timeout 600 python bench.py --no-cpu-baseline --no-e2e --stage-plan 0 --steps 10 > gpurun_out/bench_gnmt16_l2_$mb.json 2> gpurun_out/bench_gnmt16_l2_$mb.err
done
