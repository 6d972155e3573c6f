"""Boundary CTAs per side (knob boundary_ctas) for the per-iteration kernel with the static
schedule on L2-resident grids, with compute: auto split (P:400 reconstruction) vs one CTA per unit."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_baydamirlibu24_b200 as jb
from bench_latency import per_iter_us
for shape in [(128, 128, 128), (192, 192, 192), (1, 2048, 2048)]:
    for P in (2, 4, 8):
        for bc in (0, 2, 4, 8, 16):
            with jb.Jacobi(shape, virtual=P) as j:
                j.set_param("resident", 0); j.set_param("tblock", 0)
                if bc: j.set_param("boundary_ctas", bc)
                try:
                    j.run(20)
                    us = round(per_iter_us(j, 200, reps=3), 3)
                except Exception as e:
                    us = str(e)[:40]
                print(json.dumps({"shape": shape, "P": P, "boundary_ctas": bc, "us": us}), flush=True)
