"""LL vs flag halo protocol: per-iteration us of the streaming CPU-Free kernel (and the graph
baseline), virtual slabs, with and without compute."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))  # repo root
import paper_conf_sc_baydamirlibu24_b200 as jb
from bench_latency import per_iter_us
rows = []
for name, shape in {"C5a 3D 128^3": (128, 128, 128), "C5b 2D 1024^2": (1, 1024, 1024), "C2 16384^2": (1, 16384, 16384), "C3 512^3": (512, 512, 512)}.items():
    for P in (2, 4, 8):
        big = "C2" in name or "C3" in name
        with jb.Jacobi(shape, virtual=P) as j:
            j.set_param("resident", 0); j.set_param("tblock", 0)
            for label, mode, ll in [("flags", jb.MODE_CPUFREE, 0), ("LL", jb.MODE_CPUFREE, 1), ("graph", jb.MODE_BASELINE_GRAPH, 0)]:
                if big and label == "graph":
                    continue
                j.set_param("halo_ll", ll)
                for nocomp in (True, False):
                    j.set_mode(mode, jb.FLAG_NO_COMPUTE if nocomp else 0)
                    j.run(20)
                    us = per_iter_us(j, 40 if big else 400, reps=3)
                    r = {"config": name, "P": P, "proto": label, "no_compute": nocomp, "us_per_iter": round(us, 3)}
                    rows.append(r)
                    print(json.dumps(r), flush=True)
