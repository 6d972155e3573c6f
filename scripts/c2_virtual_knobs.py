"""C2 (2D 16384^2) with 8 virtual slabs, time-blocked K = 5: Gcell/s over the edge-zone / schedule
knobs vs 1 slab — where the multi-slab gap comes from."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_baydamirlibu24_b200 as jb
cells = 16382 * 16382
def rate(j, n=100):
    j.run(n); t1 = j.last_time_ms(); j.run(2 * n); t2 = j.last_time_ms()
    return cells * n / ((t2 - t1) * 1e-3) * 1e-9
for P, prm in [(1, {}), (8, {}), (8, {"boundary_ctas": 1}), (8, {"boundary_ctas": 2}), (8, {"boundary_ctas": 8}),
               (8, {"tb_min_block": 8}), (8, {"tb_min_block": 32}), (8, {"tb_min_block": 64}), (2, {}), (4, {})]:
    with jb.Jacobi((16384, 16384), virtual=P if P > 1 else 0) as j:
        for k, v in prm.items():
            j.set_param(k, v)
        j.run(10)
        r = [rate(j) for _ in range(3)]
        print(json.dumps({"P": P, "prm": prm, "gcells": round(max(r), 1), "all": [round(x, 1) for x in r]}), flush=True)
