"""Summarise PD_WAVE_PROBE output of the LSTM wavefront kernel (csrc/lstm_wave.cu):
per item visit, stamps 0 weight producer first K-block, 1 dependencies satisfied, 2 last MMA
issued, 3 accumulator ready, 4 partials exchanged (bwd) / staged (fwd), 5 published.
usage: wave_probe.py PROBE.txt   (summarises the last fwd and the last bwd launch)"""
import sys

import numpy as np


def parse(line):
    head, *ctas = line.split("|")
    rows = []
    for c in ctas:
        vis = [v.split() for v in c.split(";") if v.strip()]
        rows.append(np.array([[int(x) for x in v] for v in vis], dtype=np.float64) / 1e3)  # us
    return head.strip(), rows


def summarise(head, rows):
    print(head)
    nv = max(len(r) for r in rows)
    per = {k: [] for k in ("deps_wait", "load_mma", "mma_to_acc", "exchange_or_stage", "cell_publish", "period",
                           "w_ahead")}
    for r in rows:
        for v in range(len(r)):
            e = r[v]
            if v > 0:
                per["deps_wait"].append(e[1] - r[v - 1][5])
                per["period"].append(e[5] - r[v - 1][5])
            per["w_ahead"].append(e[1] - e[0])
            per["load_mma"].append(e[2] - e[1])
            per["mma_to_acc"].append(e[3] - e[2])
            per["exchange_or_stage"].append(e[4] - e[3])
            per["cell_publish"].append(e[5] - e[4])
            if len(e) > 7 and e[6] > 0 and e[7] > 0:
                per.setdefault("cell_loop_t0", []).append(e[6] - e[4])
                per.setdefault("epi_barrier", []).append(e[7] - e[6])
                per.setdefault("fence_publish", []).append(e[5] - e[7])
    end = max(r[-1][5] for r in rows)
    print(f"  visits/CTA {nv}, CTAs {len(rows)}, kernel span {end:.1f} us")
    for k, v in per.items():
        v = np.array([x for x in v if x > -1e5])
        if len(v):
            print(f"  {k:18s} median {np.median(v):7.2f} us  p90 {np.percentile(v, 90):7.2f}  mean {v.mean():7.2f}")


def main(path):
    lines = [l for l in open(path) if l.strip()]
    for kind in ("fwd", "bwd"):
        ls = [l for l in lines if l.startswith(kind)]
        if ls:
            summarise(*parse(ls[-1]))


if __name__ == "__main__":
    main(sys.argv[1])
