#!/usr/bin/env python
"""3D K = 3 with neighbours: throughput vs the number of boundary CTAs per side (virtual slabs
on one GPU).  Development tool: python scripts/tb3_edge_split.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_baydamirlibu24_b200 as jb  # noqa: E402

shape, cells, iters = (512, 512, 512), 510 ** 3, 99
for P in (2, 4):
    for name, prm in [("per-iteration", {"tblock": 0})] + [
            (f"K=3 boundary_ctas={bc}", {"tblock": 1, "tb_k": 3, "boundary_ctas": bc}) for bc in (-1, 8, 16, 24, 32)]:
        with jb.Jacobi(shape, virtual=P) as j:
            j.set_param("resident", 0)
            try:
                for n, v in prm.items():
                    j.set_param(n, v)
                j.run(iters)
                j.run(iters)
                d = j.describe(0)
                print(f"C3 virtual P={P} {name}: {cells * iters / j.last_time_ms() / 1e6:.1f} Gcell/s "
                      f"(n_top {d.get('n_top')}, n_bot {d.get('n_bot')}, ctas {d.get('ctas')})", flush=True)
            except jb.JacobiError as e:
                print(f"C3 virtual P={P} {name}: {e}", flush=True)
