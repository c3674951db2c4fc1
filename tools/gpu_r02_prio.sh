# MLP-4096 backward: dX chain vs dW+update contention -- stream priorities x dW grid cap
mkdir -p gpurun_out
for pr in 0 1; do for cap in 0 128 108 88; do
  PD_STREAM_PRIO=$pr PD_DW_MAX_CTAS=$cap timeout 600 python bench.py --config mlp4096 --no-cpu-baseline --no-e2e --stage-plan 0 --steps 10 > gpurun_out/bench_mlp_p${pr}_c${cap}.json 2> gpurun_out/bench_mlp_p${pr}_c${cap}.err
done; done
