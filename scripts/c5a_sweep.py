"""C5a (3D 128^3) with compute: per-iteration us of the CPU-Free kernels over their knobs, 1 and 2
virtual slabs — where the per-iteration streaming kernel's time goes on an L2-resident grid."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_baydamirlibu24_b200 as jb
from bench_latency import per_iter_us
base = {"resident": 0, "tblock": 0}
variants = [{}, {"schedule": 0}, {"schedule": 1}, {"min_block": 2}, {"min_block": 4}, {"min_block": 16},
            {"tile_y": 4}, {"tile_y": 16}, {"tile_y": 4, "min_block": 4}, {"dyn_help": 0},
            {"resident": 1}, {"resident": 1, "block_sync": 1}, {"tblock": 1}, {"ctas": 74}]
for P in (1, 2, 4):
    for v in variants:
        prm = {**base, **v}
        with jb.Jacobi((128, 128, 128), virtual=P if P > 1 else 0) as j:
            try:
                for k, x in prm.items():
                    j.set_param(k, x)
                j.run(12)
                us = round(per_iter_us(j, 150, reps=3), 3)
            except Exception as e:
                us = str(e)[:60]
            print(json.dumps({"P": P, "prm": v, "us": us}), flush=True)
