mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -rf -x -k "vgg or conv or fullsize or stash_bf16" > gpurun_out/pytest_c8.log 2>&1; echo "exit $?" >> gpurun_out/pytest_c8.log
for b in 0 1; do PD_C8_BOXES=$b timeout 600 python bench.py --config vgg16 --no-cpu-baseline --no-e2e --stage-plan 0 --steps 10 > gpurun_out/bench_vgg_c8box$b.json 2> gpurun_out/bench_vgg_c8box$b.err; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_vgg16_c8.csv -k regex:conv_c8 python bench.py --config vgg16 --no-cpu-baseline --no-e2e --stage-plan 0 --steps 1 --warmup 0 --minibatches 1 > /dev/null 2>&1
