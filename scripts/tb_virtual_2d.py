import sys; sys.path.insert(0, '.')
import paper_conf_sc_baydamirlibu24_b200 as jb
shape = (16384, 16384); cells = 16382 ** 2; iters = 200
for P in (2, 4, 8):
    for name, prm in [("per-iteration", {"tblock": 0}), ("K=5", {"tblock": 1, "tb_k": 5}), ("K=3", {"tblock": 1, "tb_k": 3, "tb_ppt": 2}), ("K=2", {"tblock": 1, "tb_k": 2})]:
        with jb.Jacobi(shape, virtual=P) as j:
            j.set_param("resident", 0)
            for n, v in prm.items(): j.set_param(n, v)
            j.run(iters); j.run(iters)
            print(f"C2 virtual P={P} {name}: {cells * iters / j.last_time_ms() / 1e6:.1f} Gcell/s (K used {j.get_param('last_tb_k')})", flush=True)
