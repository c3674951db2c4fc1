"""Per-launch DRAM traffic of an `ncu --set full` capture (raw page CSV) -> JSON that bench.py
reports as roofline.traffic.  usage: ncu_traffic.py RAW.csv KEY OUT.json [ROW] [CONFIG]
(merges into OUT.json; ROW = the launch, default 0; CONFIG = the bench config the launch came
from -- bench.py uses the record only for that config)"""
import csv
import json
import os
import sys


def main(raw, key, out, row="0", config=None):
    rows = list(csv.reader(open(raw)))
    h, units, vals = rows[0], rows[1], rows[2 + int(row)]
    col = {n: i for i, n in enumerate(h)}

    def mb(name):
        v = float(vals[col[name]].replace(",", ""))
        u = units[col[name]]
        return v * {"byte": 1e-6, "Kbyte": 1e-3, "Mbyte": 1.0, "Gbyte": 1e3}[u]

    def us(name):
        v = float(vals[col[name]].replace(",", ""))
        return v * {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3}.get(units[col[name]], 1.0)

    rec = {"kernel": vals[col["Kernel Name"]][:120], "dram_read_MB": mb("dram__bytes_read.sum"),
           "dram_write_MB": mb("dram__bytes_write.sum"),
           "duration_us": us("gpu__time_duration.sum"),
           "source": os.path.basename(raw)}
    rec["traffic_MB"] = rec["dram_read_MB"] + rec["dram_write_MB"]
    if config:
        rec["config"] = config
    d = json.load(open(out)) if os.path.exists(out) else {}
    d[key] = rec
    json.dump(d, open(out, "w"), indent=1)
    print(key, rec)


if __name__ == "__main__":
    main(*sys.argv[1:6])
