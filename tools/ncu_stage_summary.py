#!/usr/bin/env python
"""Per-stage tensor-pipe activity from the ncu launch lists of tools/gpu_ncu_r02.sh (each stage
of the 8-stage GNMT-16 plan run alone, pd_stage_solo, metrics gpu__time_duration,
sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed, dram bytes).  For every
stage: time-weighted tensor-pipe active % over all its kernels and per kernel family, and
DRAM GB/s.  ncu serialises launches and runs them cold, so absolute durations are not the
bench's; the per-kernel counters are what this table is for.
    python tools/ncu_stage_summary.py gpurun_out/stage{0..7}_ncu.csv > profiles/stage_tensor_r02.md
"""
import collections
import csv
import json
import re
import sys


def family(name):
    n = name
    if "lstm_wave_kernel" in n:
        return "lstm_wave_bwd" if re.search(r"lstm_wave_kernel<(true|1)", n) else "lstm_wave_fwd"
    if "tc_gemm_update_kernel" in n:
        return "gemm_dw_fused_update"
    if "tc_gemm_kernel" in n:
        return "gemm_tc"
    if "softmax" in n:
        return "softmax_ce"
    if "update" in n:
        return "optimizer_update"
    return "other"


def load(path):
    rows = [r for r in csv.reader(open(path)) if len(r) > 10]
    h = rows[0]
    ki, mi, ui, vi, ii = (h.index(x) for x in ("Kernel Name", "Metric Name", "Metric Unit", "Metric Value", "ID"))
    launches = collections.OrderedDict()
    for r in rows[1:]:
        d = launches.setdefault(r[ii], {"name": r[ki]})
        v = float(r[vi].replace(",", "")) if r[vi] not in ("", "n/a") else 0.0
        scale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3, "byte": 1e-9, "Kbyte": 1e-6, "Mbyte": 1e-3,
                 "Gbyte": 1.0}.get(r[ui], 1.0)
        d[r[mi]] = v * scale
    return list(launches.values())


def summarise(path):
    ls = load(path)
    fam = collections.defaultdict(lambda: [0.0, 0.0, 0.0])  # us, tensor% x us, GB
    for d in ls:
        t = d.get("gpu__time_duration.sum", 0.0)
        f = fam[family(d["name"])]
        f[0] += t
        f[1] += t * d.get("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed", 0.0)
        f[2] += d.get("dram__bytes_read.sum", 0.0) + d.get("dram__bytes_write.sum", 0.0)
    tot = sum(v[0] for v in fam.values())
    ten = sum(v[1] for v in fam.values()) / max(tot, 1e-9)
    return {"launches": len(ls), "total_us": tot, "tensor_active_pct": ten,
            "families": {k: {"us": v[0], "share": v[0] / max(tot, 1e-9), "tensor_active_pct": v[1] / max(v[0], 1e-9),
                             "dram_GBps": v[2] / max(v[0] * 1e-6, 1e-12)} for k, v in fam.items()}}


def main(paths):
    out = {}
    print("| stage | launches | ncu time (us) | tensor-pipe active (time-weighted) | wavefront fwd | wavefront bwd | GEMMs |")
    print("|---|---|---|---|---|---|---|")
    for p in paths:
        s = int(re.search(r"stage(\d+)", p).group(1))
        r = summarise(p)
        out[s] = r
        f = r["families"]
        cell = lambda k: (f"{f[k]['tensor_active_pct']:.1f} % ({f[k]['share'] * 100:.0f} % of time)" if k in f else "-")
        gem = [k for k in f if k.startswith("gemm")]
        gemt = sum(f[k]["us"] for k in gem)
        gemp = sum(f[k]["us"] * f[k]["tensor_active_pct"] for k in gem) / max(gemt, 1e-9)
        print(f"| {s} | {r['launches']} | {r['total_us']:.0f} | {r['tensor_active_pct']:.1f} % | {cell('lstm_wave_fwd')} | "
              f"{cell('lstm_wave_bwd')} | {gemp:.1f} % ({gemt / max(r['total_us'], 1e-9) * 100:.0f} % of time) |")
    json.dump(out, open(paths[0].rsplit("/", 1)[0] + "/stage_tensor.json", "w"), indent=1)


if __name__ == "__main__":
    main(sys.argv[1:])
