import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np
import oracle
import paper_conf_sc_baydamirlibu24_b200 as jb
from jacobi_inputs import u12
cases = [((24, 70), 2, {}), ((20, 70), 2, {"tb_k": 2}), ((12, 9, 33), 2, {}),
         ((12, 9, 33), 1, {}), ((12, 9, 33), 1, {"tb_k": 2}), ((30, 40), 1, {}), ((30, 40), 1, {"tb_k": 3}),
         ((30, 40), 1, {"tb_k": 5, "stages": 4}), ((30, 40), 1, {"tb_k": 2, "stages": 4}),
         ((30, 40), 1, {"tb_k": 3, "tb_ppt": 2, "stages": 4}), ((30, 40), 1, {"tb_k": 3, "tb_ppt": 4, "stages": 32}),
         ((30, 600), 1, {"tb_k": 3, "tb_ppt": 4}), ((30, 50, 140), 1, {}), ((26, 50, 140), 2, {"tb_k": 3})]
shape, P, prm = cases[int(sys.argv[1])]
f = u12(shape, 4)
with jb.Jacobi(shape, virtual=P) if P > 1 else jb.Jacobi(shape) as j:
    j.set_param("tblock", 1); j.set_param("resident", 0)
    for k, v in prm.items(): j.set_param(k, v)
    j.scatter(f); j.run(8)
    print("CASE", sys.argv[1], "K", j.get_param("last_tb_k"), "OK" if np.array_equal(j.gather(), oracle.jacobi(f, 8)) else "MISMATCH")
