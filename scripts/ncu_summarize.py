#!/usr/bin/env python
"""Per-iteration DRAM traffic of the CPU-Free kernels from `ncu --set full` raw CSV exports
(scripts/profile_round.sh) -> profiles/ncu_summary.json, read by bench.py for roofline.traffic.

    python scripts/ncu_summarize.py NAME=RAW_CSV:ALG_BYTES_PER_ITER[:ITERS] ...
"""
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def raw_metrics(path):
    rows = list(csv.reader(open(path)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    return {h: (v, u) for h, u, v in zip(hdr, units, vals)}


def num(d, k, scale_units=True):
    v, u = d[k]
    x = float(v.replace(",", ""))
    if scale_units:
        x *= {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
              "nsecond": 1e-6, "usecond": 1e-3, "msecond": 1.0, "second": 1e3}.get(u, 1)
    return x


def main():
    out_path = os.path.join(ROOT, "profiles", "ncu_summary.json")
    summary = json.load(open(out_path)) if os.path.exists(out_path) else {}
    for arg in sys.argv[1:]:
        name, spec = arg.split("=", 1)
        parts = spec.split(":")
        path, alg = parts[0], float(parts[1])
        iters = int(parts[2]) if len(parts) > 2 else 20
        d = raw_metrics(path)
        rd, wr = num(d, "dram__bytes_read.sum"), num(d, "dram__bytes_write.sum")
        ms = num(d, "gpu__time_duration.sum")
        summary[name] = {
            "kernel": d["Kernel Name"][0].split("(")[0].replace("void <unnamed>::", ""),
            "iters_per_launch": iters,
            "dram_bytes_per_iter": (rd + wr) / iters,
            "dram_read_per_iter": rd / iters,
            "dram_write_per_iter": wr / iters,
            "alg_bytes_per_iter": alg,
            "traffic_over_alg": (rd + wr) / iters / alg,
            "ms_per_iter_under_ncu": ms / iters,
            "dram_gbs_under_ncu": (rd + wr) / (ms / 1e3) / 1e9,
            "registers": int(num(d, "launch__registers_per_thread", False)),
            "source": f"profiles/{os.path.basename(path)} (ncu --set full --clock-control none, 1 launch of {iters} iterations)",
        }
    json.dump(summary, open(out_path, "w"), indent=1)
    print(json.dumps(summary, indent=1))


if __name__ == "__main__":
    main()
