#!/usr/bin/env python
"""Edge-zone cost of the time-blocked kernels with VIRTUAL slabs on one GPU (P slab groups of
CTAs, the full flag/halo protocol): C2 (2D K = 5) and C3 (3D K = 3) vs the per-iteration kernel
and vs one slab.  Development tool (GPU box): python scripts/edge_zone_bench.py [--iters N]."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_sc_baydamirlibu24_b200 as jb  # noqa: E402


def rate(shape, P, prm, iters, reps=3):
    cells = (shape[-1] - 2) * (shape[-2] - 2) * (shape[0] - 2 if len(shape) == 3 else 1)
    with (jb.Jacobi(shape, virtual=P) if P > 1 else jb.Jacobi(shape)) as j:
        j.set_param("resident", 0)
        for n, v in prm.items():
            j.set_param(n, v)
        j.run(iters)
        t = min((j.run(iters), j.last_time_ms())[1] for _ in range(reps))
        return cells * iters / t / 1e6, j.get_param("last_tb_k"), j.get_param("last_tblock")


def main():
    iters = int(sys.argv[sys.argv.index("--iters") + 1]) if "--iters" in sys.argv else 200
    rows = []
    for name, shape, k in [("C2", (16384, 16384), 5), ("C3", (512, 512, 512), 3)]:
        it = iters - iters % k
        for P in (1, 2, 4, 8):
            for kname, prm in [("per-iteration", {"tblock": 0}), (f"K={k}", {"tblock": 1, "tb_k": k})]:
                v, kk, tb = rate(shape, P, prm, it)
                r = {"config": name, "P": P, "kernel": kname, "gcells": round(v, 1), "K_used": kk, "tb_iters": tb}
                rows.append(r)
                print(json.dumps(r), flush=True)


if __name__ == "__main__":
    main()
