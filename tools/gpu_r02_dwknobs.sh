mkdir -p gpurun_out
for u in 2 8 4; do
  PD_DW_UNITS_C8=$u timeout 600 python bench.py --config vgg16 --no-cpu-baseline --no-e2e --stage-plan 0 --steps 10 > gpurun_out/bench_vgg_c8_$u.json 2> gpurun_out/bench_vgg_c8_$u.err
done
