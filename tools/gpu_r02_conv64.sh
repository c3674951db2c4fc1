mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -rf -x -k "vgg or conv or fullsize" > gpurun_out/pytest_conv64.log 2>&1; echo "exit $?" >> gpurun_out/pytest_conv64.log
for cg in 2 1; do PD_GEMM_CG=$cg timeout 600 python bench.py --config vgg16 --no-cpu-baseline --no-e2e --stage-plan 0 --steps 10 > gpurun_out/bench_vgg_cg$cg.json 2>/dev/null; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_conv64.csv -k regex:tc_gemm_kernel python bench.py --config vgg16 --no-cpu-baseline --no-e2e --stage-plan 0 --steps 1 --warmup 0 --minibatches 1 > /dev/null 2>&1
