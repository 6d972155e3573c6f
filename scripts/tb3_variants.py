#!/usr/bin/env python
"""3D time-blocked kernel variants (K = 3: pairs per lane, rows per warp): bitwise check against
the oracle on small ragged grids (1 slab and virtual slabs), then C3 throughput per variant.
Development tool (GPU box): python scripts/tb3_variants.py [--quick]."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import paper_conf_sc_baydamirlibu24_b200 as jb  # noqa: E402
from jacobi_inputs import u12  # noqa: E402

VARIANTS = [(3, 1, 2), (3, 1, 3)]  # (K, ppt, rows per warp)


def params(k, ppt, rpw):
    p = {"tblock": 1, "resident": 0, "tb_k": k, "tb_ppt": ppt}
    if rpw > 0:
        p["tb_rpw"] = rpw
    return p


def check():
    bad = 0
    for k, ppt, rpw in VARIANTS:
        for shape, iters, virtual in [((10, 13, 70), 7, 0), ((20, 37, 130), 9, 0), ((9, 17, 300), 6, 0),
                                      ((40, 9, 8), 5, 0), ((3, 3, 3), 4, 0), ((12, 70, 61), 10, 0),
                                      ((30, 25, 66), 13, 2), ((40, 30, 140), 12, 3)]:
            f = u12(shape, 5)
            with jb.Jacobi(shape, virtual=virtual) as j:
                for n, v in params(k, ppt, rpw).items():
                    j.set_param(n, v)
                j.scatter(f)
                j.run(iters)
                got, kk, tb = j.gather(), j.get_param("last_tb_k"), j.get_param("last_tblock")
            exp = oracle.jacobi(f, iters)
            n = int(np.count_nonzero(got.view(np.uint64) != exp.view(np.uint64)))
            print(f"K={k} ppt={ppt} rpw={rpw} {shape} it={iters} P={virtual or 1}: K used {kk} tb_iters={tb} "
                  f"{'OK' if n == 0 else f'MISMATCH {n} cells'}", flush=True)
            bad += n != 0
    return bad


def timing(iters=201):
    shape = (512, 512, 512)
    cells = 510 ** 3
    with jb.Jacobi(shape) as j:
        j.set_param("tblock", 0)
        j.run(iters)
        j.run(iters)
        print(f"C3 per-iteration kernel: {cells * iters / j.last_time_ms() / 1e6:.1f} Gcell/s", flush=True)
    for k, ppt, rpw in VARIANTS:
        with jb.Jacobi(shape) as j:
            for n, v in params(k, ppt, rpw).items():
                j.set_param(n, v)
            j.run(iters)
            ts = []
            for _ in range(3):
                j.run(iters)
                ts.append(j.last_time_ms())
            t = min(ts)
            print(f"C3 K={k} ppt={ppt} rpw={rpw}: {cells * iters / t / 1e6:.1f} Gcell/s ({t / iters * 1e3:.1f} us/iter, "
                  f"K used {j.get_param('last_tb_k')}, tb_iters {j.get_param('last_tblock')})", flush=True)


def timing_virtual(iters=201):
    shape = (512, 512, 512)
    cells = 510 ** 3
    for P in (2, 4, 8):
        for name, prm in [("per-iteration", {"tblock": 0}), ("K=3 rpw=2", {"tblock": 1, "tb_k": 3, "tb_ppt": 1, "tb_rpw": 2}),
                          ("K=2", {"tblock": 1, "tb_k": 2})]:
            with jb.Jacobi(shape, virtual=P) as j:
                j.set_param("resident", 0)
                for n, v in prm.items():
                    j.set_param(n, v)
                j.run(iters)
                j.run(iters)
                print(f"C3 virtual P={P} {name}: {cells * iters / j.last_time_ms() / 1e6:.1f} Gcell/s", flush=True)


if __name__ == "__main__":
    b = check()
    print("mismatching cases:", b, flush=True)
    if "--quick" not in sys.argv:
        timing()
        timing_virtual()
