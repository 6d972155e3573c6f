#!/usr/bin/env python
"""Time-blocked kernel variants (K iterations per HBM pass, pairs per thread): bitwise check
against the oracle on small ragged grids (1 slab and virtual slabs), then C2 throughput per
variant.  Development tool (GPU box): python scripts/tb_variants.py [--quick]."""
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import paper_conf_sc_baydamirlibu24_b200 as jb  # noqa: E402
from jacobi_inputs import u12  # noqa: E402

VARIANTS = [(5, 1, 1), (5, 1, 2), (3, 1, 2)]


def run(shape, iters, k, ppt, lag, virtual=0, extra=None):
    with jb.Jacobi(shape, virtual=virtual) as j:
        for n, v in {"tblock": 1, "resident": 0, "tb_k": k, "tb_ppt": ppt, "tb_lag": lag, **(extra or {})}.items():
            j.set_param(n, v)
        f = u12(shape, 3)
        j.scatter(f)
        j.run(iters)
        return f, j.gather(), j.get_param("last_tb_k"), j.get_param("last_tblock")


def check():
    bad = 0
    for k, ppt, lag in VARIANTS:
        for shape, iters, virtual in [((40, 3000), 15, 0), ((70, 2051), 11, 0), ((300, 130), 10, 0), ((5, 4100), 7, 0),
                                      ((3, 3), 5, 0), ((1000, 37), 20, 0), ((97, 1990), 15, 2), ((130, 2200), 30, 3),
                                      ((64, 1500), 20, 5)]:
            f, got, kk, tb = run(shape, iters, k, ppt, lag, virtual)
            exp = oracle.jacobi(f, iters)
            same = np.array_equal(got.view(np.uint64), exp.view(np.uint64))
            n = int(np.count_nonzero(got.view(np.uint64) != exp.view(np.uint64)))
            print(f"K={k} ppt={ppt} lag={lag} {shape} it={iters} P={virtual or 1}: used K={kk} tb_iters={tb} "
                  f"{'OK' if same else f'MISMATCH {n} cells'}", flush=True)
            bad += not same
    return bad


def timing(iters=200):
    shape = (16384, 16384)
    cells = (shape[0] - 2) * (shape[1] - 2)
    for k, ppt, lag in VARIANTS:
        for mb in (16, 32):
            with jb.Jacobi(shape) as j:
                for n, v in {"tblock": 1, "resident": 0, "tb_k": k, "tb_ppt": ppt, "tb_lag": lag,
                             "tb_min_block": mb}.items():
                    j.set_param(n, v)
                j.run(iters)
                ts = []
                for _ in range(3):
                    j.run(iters)
                    ts.append(j.last_time_ms())
                t = min(ts)
                print(f"C2 K={k} ppt={ppt} lag={lag} min_block={mb}: {cells * iters / t / 1e6:.1f} Gcell/s "
                      f"({t / iters * 1e3:.1f} us/iter, K used {j.get_param('last_tb_k')})", flush=True)


if __name__ == "__main__":
    b = check()
    print("mismatching cases:", b, flush=True)
    if "--quick" not in sys.argv:
        timing()
