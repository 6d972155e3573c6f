"""Interior schedule of the per-iteration streaming kernel (knob schedule: 0 static linear,
1 static lockstep, 2 dynamic guided) vs the time-blocked / resident kernels, with compute, across
grid sizes and virtual slab counts: where static schedules win (small, L2-resident slabs)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_baydamirlibu24_b200 as jb
from bench_latency import per_iter_us
shapes = [(128, 128, 128), (192, 192, 192), (256, 256, 256), (384, 384, 384), (1, 1024, 1024), (1, 2048, 2048), (1, 4096, 4096)]
for shape in shapes:
    cells = (shape[0] - 2 if shape[0] > 1 else 1) * (shape[1] - 2) * (shape[2] - 2)
    n = max(30, min(600, int(3e9 / cells / 16)))  # ~ a few ms per run
    n = n // 30 * 30
    for P in (1, 2, 4, 8):
        rows = [("auto", {})] + [(f"stream s{s}", {"resident": 0, "tblock": 0, "schedule": s}) for s in (0, 1, 2)]
        rows += [("stream s1 ty16", {"resident": 0, "tblock": 0, "schedule": 1, "tile_y": 16})] if shape[0] > 1 else []
        rows += [("tblock", {"resident": 0, "tblock": 1})]
        for label, prm in rows:
            with jb.Jacobi(shape, virtual=P if P > 1 else 0) as j:
                try:
                    for k, x in prm.items():
                        j.set_param(k, x)
                    j.run(30)
                    us = round(per_iter_us(j, n, reps=3), 3)
                    kern = ("tblock" if j.get_param("last_tblock") else "resident" if j.get_param("last_resident")
                            else "cluster" if j.get_param("last_cluster") else "stream")
                except Exception as e:
                    us, kern = str(e)[:50], "-"
                print(json.dumps({"shape": shape, "P": P, "variant": label, "kernel": kern, "us": us,
                                  "gcells": round(cells / us * 1e-3, 1) if isinstance(us, float) else None}), flush=True)
