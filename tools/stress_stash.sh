mkdir -p gpurun_out
FS=paper_conf_sosp_narayananhpsdgg19_b200/build/fault_stash/libpipedream.so
for i in $(seq 1 25); do
  for lib in main fault; do
    if [ $lib = fault ]; then export PD_LIBRARY=$FS; else unset PD_LIBRARY; fi
    timeout -s KILL 100 python tests/stash_cases.py mlp256 > gpurun_out/st_${lib}_$i.log 2>&1
    rc=$?
    echo "$lib $i rc=$rc" >> gpurun_out/stress_summary.txt
    if [ $rc -ne 0 ]; then tail -40 gpurun_out/st_${lib}_$i.log > gpurun_out/stuck_${lib}_$i.log; nvidia-smi >> gpurun_out/stuck_${lib}_$i.log; fi
    rm -f gpurun_out/st_${lib}_$i.log
  done
done
