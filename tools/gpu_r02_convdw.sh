# conv weight-gradient tile width: parity of the VGG paths, then VGG-16 bench + launch list
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -rf -x -k "vgg or conv or fullsize or stash" > gpurun_out/pytest_convdw.log 2>&1; echo "exit $?" >> gpurun_out/pytest_convdw.log
timeout 600 python bench.py --config vgg16 --no-cpu-baseline --stage-plan 0 > gpurun_out/bench_vgg16_bn256.json 2> gpurun_out/bench_vgg16_bn256.err
timeout 900 ncu --metrics gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none --csv --log-file gpurun_out/launches_vgg16_bn256.csv python bench.py --config vgg16 --no-cpu-baseline --no-e2e --stage-plan 0 --steps 1 --warmup 1 --minibatches 1 > /dev/null 2>&1
