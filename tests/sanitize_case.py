"""Tiny runs of every kernel family for compute-sanitizer (tests/test_gpu_sanitizer.py)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import oracle  # noqa: E402
import paper_conf_sc_baydamirlibu24_b200 as jb  # noqa: E402
from jacobi_inputs import u12  # noqa: E402

ok = True
for shape, P in [((20, 70), 2), ((8, 9, 33), 2), ((30, 40), 1)]:
    f = u12(shape, 3)
    for params, mode in [({"resident": 0}, jb.MODE_CPUFREE), ({"resident": 1}, jb.MODE_CPUFREE),
                         ({}, jb.MODE_BASELINE_MEMCPY), ({}, jb.MODE_BASELINE_P2P),
                         ({"resident": 0, "norm_every": 2}, jb.MODE_CPUFREE),
                         ({"resident": 0, "tblock": 0, "halo_ll": 1}, jb.MODE_CPUFREE)]:  # LL halos
        with jb.Jacobi(shape, virtual=P) if P > 1 else jb.Jacobi(shape) as j:
            for k, v in params.items():
                j.set_param(k, v)
            j.set_mode(mode)
            j.scatter(f)
            j.run(3)
            ok &= bool(np.array_equal(j.gather(), oracle.jacobi(f, 3)))
# time-blocked kernel (2D K = 5 / 3 / 2, 3D K = 3 / 2, with and without neighbours): TMA ring
# and TMA boxes, shuffles, the 3D shared-memory row exchange, edge zones; rings short enough to
# wrap inside an item (stages=4, and K = 3 with 4 pairs per lane: 14 KB stages)
for shape, P, prm in [((24, 70), 2, {}), ((20, 70), 2, {"tb_k": 2}), ((12, 9, 33), 2, {}),
                      ((12, 9, 33), 1, {}), ((12, 9, 33), 1, {"tb_k": 2}), ((30, 40), 1, {}),
                      ((30, 40), 1, {"tb_k": 3}), ((30, 40), 1, {"tb_k": 5, "tb_ppt": 2}),
                      ((30, 40), 1, {"stages": 4}), ((30, 40), 1, {"tb_k": 2, "stages": 4}),
                      # without the warp-specialised register split (the default uses it for
                      # 2D K = 5 and 3D K = 3), and 3D edge zones between virtual slabs
                      ((30, 40), 1, {"tb_ws": 0}), ((24, 70), 2, {"tb_ws": 0}), ((12, 9, 33), 1, {"tb_ws": 0}),
                      ((16, 9, 33), 2, {"tb_ws": 0})]:
    f = u12(shape, 4)
    with jb.Jacobi(shape, virtual=P) if P > 1 else jb.Jacobi(shape) as j:
        j.set_param("tblock", 1)
        j.set_param("resident", 0)
        for k, v in prm.items():
            j.set_param(k, v)
        j.scatter(f)
        j.run(8)
        ok &= bool(np.array_equal(j.gather(), oracle.jacobi(f, 8)))
# one-cluster kernel (DSMEM halo rows, cluster barriers), 16- and small clusters
for shape in [(30, 40), (5, 70), (40, 13)]:
    f = u12(shape, 5)
    with jb.Jacobi(shape) as j:
        j.set_param("cluster", 1)
        j.scatter(f)
        j.run(6)
        ok &= bool(np.array_equal(j.gather(), oracle.jacobi(f, 6)))
print("SANITIZE_CASE_OK" if ok else "SANITIZE_CASE_MISMATCH")
