"""Edge-zone A/B: Gcell/s of the time-blocked kernel with virtual slabs (where the edge zones'
share is largest) for the library named by JACOBI_LIB; one JSON line per case."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import paper_conf_sc_baydamirlibu24_b200 as jb
import oracle
from jacobi_inputs import u12
lib = os.environ.get("JACOBI_LIB", "default")
# quick parity: small grids, every slab count, forced time-blocked
ok = True
for shape, P in [((66, 300), 4), ((23, 20, 70), 2), ((40, 30, 50), 4)]:
    f = u12(shape, 3)
    with jb.Jacobi(shape, virtual=P) as j:
        j.set_param("resident", 0); j.set_param("tblock", 1)
        j.scatter(f); j.run(30)
        ok &= bool(np.array_equal(j.gather().view(np.uint64), oracle.jacobi(f, 30).view(np.uint64)))
for shape, P, n in [((16384, 16384), 1, 100), ((512, 512, 512), 1, 60), ((16384, 16384), 8, 100), ((16384, 16384), 4, 100), ((512, 512, 512), 2, 60),
                    ((512, 512, 512), 4, 60), ((512, 512, 512), 8, 60)]:
    cells = np.prod([s - 2 for s in shape])
    with jb.Jacobi(shape, virtual=P if P > 1 else 0) as j:
        j.set_param("tblock", 1)
        j.run(n // 2)
        best = 0
        for _ in range(3):
            j.run(n); t1 = j.last_time_ms(); j.run(2 * n); t2 = j.last_time_ms()
            best = max(best, cells * n / ((t2 - t1) * 1e-3) * 1e-9)
    print(json.dumps({"lib": os.path.basename(lib), "shape": shape, "P": P, "gcells": round(best, 1), "parity": ok}), flush=True)
