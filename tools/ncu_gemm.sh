#!/bin/bash
# kernel durations (ncu, serialized) for the MLP small-M GEMM configurations
for cfg in "1 64 1" "2 128 1" "2 256 1" "2 256 2" "2 256 4" "1 256 4"; do
  set -- $cfg
  PD_GEMM_CG=$1 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ng_$1_$2_$3.csv python tools/gemm_bench.py fwd $2 $3 > /dev/null 2>&1
  python - "$cfg" gpurun_out/ng_$1_$2_$3.csv <<'PY'
import csv, sys, collections
rows=[r for r in csv.reader(open(sys.argv[2])) if len(r)>10 and r[0]!='ID']
agg=collections.defaultdict(list)
for r in rows:
    n=r[4].split('(')[0].replace('void ','').replace('pd::<unnamed>::','')[:40]
    if 'pd::' in r[4] or 'tc_gemm' in n or 'splitk' in n:
        agg[n].append(float(r[-1])/1e3)
print(sys.argv[1], {k: round(sorted(v)[len(v)//2],2) for k,v in agg.items()})
PY
done
