# overlapped LSTM weight gradients: parity, then GNMT-16 per-stage table with / without
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_lstm_rec.py -q -rf -x -k "overlapped or wavefront_matches" > gpurun_out/pytest_wavedw.log 2>&1; echo "exit $?" >> gpurun_out/pytest_wavedw.log
for s in 5 1; do for ov in 1 0; do PD_WAVE_DW=$ov timeout 300 python bench.py --stage $s --solo-runs 3 > gpurun_out/stage${s}_dw$ov.json 2> gpurun_out/stage${s}_dw$ov.err; done; done
