"""No-compute CPU-Free iteration cost vs the number of CTAs per slab (knob ctas), C5b 2D 1024^2,
1 and 2 virtual slabs: how much of the per-iteration floor is the grid barrier's CTA count."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_baydamirlibu24_b200 as jb
from bench_latency import per_iter_us
for P in (1, 2):
    for ctas in (4, 16, 64, 148):
        with jb.Jacobi((1, 1024, 1024), virtual=P if P > 1 else 0) as j:
            j.set_param("resident", 0); j.set_param("tblock", 0); j.set_param("ctas", ctas)
            j.set_mode(jb.MODE_CPUFREE, jb.FLAG_NO_COMPUTE)
            try:
                j.run(20)
                us = per_iter_us(j, 400, reps=5)
            except Exception as e:
                us = str(e)
            print(json.dumps({"P": P, "ctas": ctas, "us_per_iter": us}), flush=True)
