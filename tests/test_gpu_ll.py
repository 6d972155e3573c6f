"""GPU parity of the LL halo protocol (knob "halo_ll") of the streaming CPU-Free
kernel: halo cells travel as tagged 16-byte LL cells, polled by the receiver, instead of plain
stores + a sys-scope release flag.  The field must stay bit-identical to the oracle for every slab
count and run split (decomposition invariance; every iteration reads the previous
time step), runs of every kernel must mix (the first / last halo of an LL run use the flag
protocol, so flags and halo planes are valid between runs), and a neighbour that never sends
must still end in the watchdog, not a hang.
"""
import numpy as np
import pytest

import oracle
import paper_conf_sc_baydamirlibu24_b200 as jb
from jacobi_inputs import u12

pytestmark = pytest.mark.gpu


def assert_bitwise(got, exp, what=""):
    if not np.array_equal(np.asarray(got).view(np.uint64), np.asarray(exp).view(np.uint64)):
        n = int(np.count_nonzero(np.asarray(got).view(np.uint64) != np.asarray(exp).view(np.uint64)))
        raise AssertionError(f"{what}: {n} cells differ")


def ll_handle(shape, virtual, **params):
    j = jb.Jacobi(shape, virtual=virtual)
    for k, v in {"resident": 0, "tblock": 0, "halo_ll": 1, **params}.items():
        j.set_param(k, v)
    return j


@pytest.mark.parametrize("shape", [(20, 64), (131, 700), (67, 2100), (11, 9, 40), (30, 25, 66), (40, 70, 130)])
@pytest.mark.parametrize("P", [2, 3, 4])
@pytest.mark.parametrize("iters", [1, 2, 7, 20])
def test_ll_vs_oracle(shape, P, iters):
    if (shape[0] - 2) // P < 2:
        pytest.skip("slab too thin")
    f = u12(shape, 11)
    with ll_handle(shape, P) as j:
        j.scatter(f)
        j.run(iters)
        got = j.gather()
    assert_bitwise(got, oracle.jacobi(f, iters), f"LL {shape} P={P} it={iters}")


@pytest.mark.parametrize("shape", [(131, 700), (30, 25, 66)])
def test_ll_runs_mix_with_every_kernel(shape):
    """LL runs, flag-protocol runs, time-blocked runs and the resident kernel alternate on one
    handle: run(a); run(b) == run(a + b) whatever kernel each run used."""
    f = u12(shape, 12)
    P = 3
    total = 0
    with ll_handle(shape, P) as j:
        j.scatter(f)
        for params, n in [({}, 5), ({"halo_ll": 0}, 4), ({}, 6), ({"tblock": 1}, 7), ({}, 3),
                          ({"resident": -1, "tblock": 0}, 5), ({"resident": 0}, 9), ({}, 1), ({}, 2)]:
            for k, v in params.items():
                j.set_param(k, v)
            j.run(n)
            total += n
            if "halo_ll" in params:
                j.set_param("halo_ll", 1)
        got = j.gather()
    assert_bitwise(got, oracle.jacobi(f, total), f"mixed runs {shape}")


def test_ll_scatter_between_runs():
    """A scatter between LL runs: the iteration counter keeps growing, so the LL cells left by the
    earlier run (older tags) are never taken for the new run's halos."""
    shape = (131, 700)
    f1, f2 = u12(shape, 13), u12(shape, 14)
    with ll_handle(shape, 3) as j:
        j.scatter(f1)
        j.run(6)
        j.scatter(f2)
        j.run(5)
        got = j.gather()
    assert_bitwise(got, oracle.jacobi(f2, 5), "scatter between LL runs")


@pytest.mark.parametrize("shape", [(20, 64), (11, 9, 40)])
def test_ll_no_compute_halo_slots_hold_neighbour_edges(shape):
    """No-compute mode with LL cells: after the run every halo plane holds the
    neighbour's edge plane, as with the flag protocol."""
    f = u12(shape, 4)
    P = 3
    with ll_handle(shape, P) as j:
        j.scatter(f)
        j.set_mode(jb.MODE_CPUFREE, jb.FLAG_NO_COMPUTE).run(5)
        par = j.iterations & 1
        slabs = [j.read_slab(i, par) for i in range(P)]
        chunks = [j.describe(i)["chunk"] for i in range(P)]
        j.set_mode(jb.MODE_CPUFREE, 0)
        j.scatter(f)
        j.run(4)  # compute after no-compute runs on the same handle
        got = j.gather()
    for g in range(P):
        if g > 0:
            assert np.array_equal(slabs[g][0], slabs[g - 1][chunks[g - 1]])
        if g < P - 1:
            assert np.array_equal(slabs[g][chunks[g] + 1], slabs[g + 1][1])
    assert_bitwise(got, oracle.jacobi(f, 4), "compute after LL no-compute")


def test_ll_watchdog_timeout_without_hang():
    """Slab 0 never sends (FLAG_DROP_SIGNAL): its neighbour's LL poll ends in the watchdog."""
    with ll_handle((40, 200), 2) as j:
        j.set_param("timeout_ms", 300)
        j.set_mode(jb.MODE_CPUFREE, jb.FLAG_DROP_SIGNAL)
        with pytest.raises(jb.JacobiError) as e:
            j.run(10)
        assert e.value.code == jb.JACOBI_ETIMEOUT
    f = u12((40, 200), 1)
    with ll_handle(f.shape, 2) as j:
        j.scatter(f)
        j.run(3)
        assert_bitwise(j.gather(), oracle.jacobi(f, 3), "after LL timeout")


def test_ll_with_norm_runs_keeps_flags():
    """The norm kernel (N4) keeps the flag protocol even with halo_ll = 1 (a convergence stop
    can end a run at any iteration); fields stay bitwise and the stop iteration exact."""
    shape = (67, 300)
    f = u12(shape, 15)
    with ll_handle(shape, 3) as j:
        j.scatter(f)
        j.set_tolerance(0.0, 5)  # (tolerance 0: the run never stops early)
        j.run(10)
        j.set_param("norm_every", 0)
        j.run(7)
        got = j.gather()
    assert_bitwise(got, oracle.jacobi(f, 17), "norm + LL")
