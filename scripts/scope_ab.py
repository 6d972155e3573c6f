"""Halo-flag scope A/B: per-iteration us of the CPU-Free kernels with virtual
slabs, flags released / acquired at .sys scope (flag_scope = 0, the scope a neighbour on another GPU
needs) vs .gpu scope (flag_scope = -1 auto for virtual slabs), with and without compute; the CUDA
graph baseline beside it.  Every CPU-Free run with compute is checked bitwise against the 1-slab
result of the same grid.  Usage: python scripts/scope_ab.py [--out file.jsonl]"""
import argparse
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))  # repo root
import paper_conf_sc_baydamirlibu24_b200 as jb  # noqa: E402
from bench_latency import per_iter_us  # noqa: E402
from jacobi_inputs import u12  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--out", default="")
ap.add_argument("--slabs", default="2,4,8")
args = ap.parse_args()
rows = []
out = open(args.out, "w") if args.out else None
for name, shape in {"C5a 3D 128^3": (128, 128, 128), "C5b 2D 1024^2": (1, 1024, 1024)}.items():
    f = u12(shape if shape[0] > 1 else shape[1:], 7)
    with jb.Jacobi(shape) as j1:
        j1.scatter(f)
        j1.run(30)
        ref = j1.gather()
    for P in [int(s) for s in args.slabs.split(",")]:
        with jb.Jacobi(shape, virtual=P) as j:
            for label, mode, scope in [("cpufree_sys", jb.MODE_CPUFREE, 0), ("cpufree_gpu", jb.MODE_CPUFREE, -1),
                                       ("graph", jb.MODE_BASELINE_GRAPH, -1)]:
                j.set_param("flag_scope", scope)
                for nocomp in (True, False):
                    j.set_mode(mode, jb.FLAG_NO_COMPUTE if nocomp else 0)
                    ok = None
                    if not nocomp and mode == jb.MODE_CPUFREE:
                        j.scatter(f)
                        j.run(30)
                        ok = bool(np.array_equal(j.gather().view(np.uint64), ref.view(np.uint64)))
                    j.run(20)
                    us = per_iter_us(j, 400, reps=5)
                    kern = ("tblock" if j.get_param("last_tblock") else "resident" if j.get_param("last_resident")
                            else "stream") if mode == jb.MODE_CPUFREE else "-"
                    r = {"config": name, "P": P, "variant": label, "no_compute": nocomp, "kernel": kern,
                         "us_per_iter": round(us, 3), "bitwise_vs_1slab": ok}
                    rows.append(r)
                    print(json.dumps(r), flush=True)
                    if out:
                        out.write(json.dumps(r) + "\n")
                        out.flush()
