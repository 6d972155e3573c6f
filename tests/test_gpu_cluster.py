"""GPU parity of the one-cluster on-chip kernel (cluster.cu, knob "cluster"): a
single 2D slab kept in the shared memory of one thread-block cluster, halo rows between its CTAs
through DSMEM, one hardware cluster barrier per iteration (the device-side iteration barrier of
P:372 at cluster scope).  Bit-identical to the oracle (same operation order, no contraction) for
ragged shapes and every run split, mixing with every other kernel, and loud (EINVAL) where it
does not apply.
"""
import numpy as np
import pytest

import oracle
import paper_conf_sc_baydamirlibu24_b200 as jb
from jacobi_inputs import SEED_BENCH, u12

pytestmark = pytest.mark.gpu


def assert_bitwise(got, exp, what=""):
    g, e = np.asarray(got).view(np.uint64), np.asarray(exp).view(np.uint64)
    if not np.array_equal(g, e):
        raise AssertionError(f"{what}: {int(np.count_nonzero(g != e))} cells differ")


@pytest.mark.parametrize("shape", [(3, 3), (4, 9), (10, 12), (18, 1000), (64, 96), (129, 131), (256, 256),
                                   (255, 257), (300, 131), (40, 700)])
@pytest.mark.parametrize("iters", [1, 2, 7, 40])
def test_cluster_vs_oracle(shape, iters):
    f = u12(shape, 21)
    with jb.Jacobi(shape) as j:
        j.set_param("cluster", 1)
        j.scatter(f)
        j.run(iters)
        assert j.get_param("last_cluster") in (1, 2, 4, 8, 16)
        got = j.gather()
    assert_bitwise(got, oracle.jacobi(f, iters), f"cluster {shape} it={iters}")


def test_cluster_c1_1000_iterations():
    """BASELINE config C1 (2D 256x256, 1000 iterations, 1 GPU) on the cluster kernel vs the oracle."""
    f = u12((256, 256), SEED_BENCH)
    with jb.Jacobi((256, 256)) as j:
        j.set_param("cluster", 1)
        j.run(1000)
        got = j.gather()
    assert_bitwise(got, oracle.jacobi(f, 1000, 8), "C1 cluster")


def test_cluster_runs_mix_with_every_kernel():
    shape = (200, 300)
    f = u12(shape, 22)
    total = 0
    with jb.Jacobi(shape) as j:
        j.scatter(f)
        for params, n in [({"cluster": 1}, 5), ({"cluster": 0, "tblock": 1}, 10), ({"cluster": 1, "tblock": -1}, 3),
                          ({"cluster": 0, "tblock": 0, "resident": 1}, 4), ({"cluster": 1}, 1),
                          ({"cluster": 0, "tblock": 0, "resident": 0}, 6), ({"cluster": 1, "resident": -1}, 8)]:
            for k, v in params.items():
                j.set_param(k, v)
            j.run(n)
            total += n
        got = j.gather()
    assert_bitwise(got, oracle.jacobi(f, total), "mixed kernels")


def test_cluster_not_applicable_is_loud():
    for shape, virtual in [((10, 12, 14), 0), ((40, 64), 2), ((4096, 4096), 0)]:
        with jb.Jacobi(shape, virtual=virtual) as j:
            j.set_param("cluster", 1)
            with pytest.raises(jb.JacobiError) as e:
                j.run(2)
            assert e.value.code == jb.JACOBI_EINVAL
    with jb.Jacobi((64, 64)) as j:  # no-compute runs are not for this kernel either
        j.set_param("cluster", 1)
        j.set_mode(jb.MODE_CPUFREE, jb.FLAG_NO_COMPUTE)
        with pytest.raises(jb.JacobiError):
            j.run(2)
