"""GPU edge cases of the boundary: empty batches, zero-length runs, degenerate and maximum sizes,
argument errors -- each compared with the oracle where there is a result."""
import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def lib():
    import torch

    assert torch.cuda.is_available()
    import paper_conf_ipps_awasthillw16_b200 as m

    return m


@pytest.mark.parametrize("n", [1, 10, 1000])
@pytest.mark.parametrize("problem", ["cdd", "ucddcp"])
def test_empty_batch(lib, n, problem):
    import torch

    inst = gen.ucddcp_instance(n, 1) if problem == "ucddcp" else gen.cdd_instance(n, 1, 0.4)
    ins = lib.Instance.from_gen(inst)
    fn = lib.ucddcp_eval_batch if problem == "ucddcp" else lib.cdd_eval_batch
    ld = (n + 7) // 8 * 8
    out = fn(ins, torch.empty((0, ld), dtype=torch.int16, device="cuda"))
    torch.cuda.synchronize()
    assert out.shape == (0,)
    lib.cdd_check(ins)  # no data-error flag, no CUDA error


@pytest.mark.parametrize("n,chains,lanes", [(1, 5, 0), (2, 40, 0), (50, 300, 8), (1000, 64, 0)])
def test_sa_zero_steps_is_best_initial_state(lib, n, chains, lanes):
    # Alg. 1 with no iterations returns the best of the random initial states (R13, R14)
    import torch

    inst = gen.cdd_instance(n, 2, 0.6)
    ins = lib.Instance.from_gen(inst)
    res = lib.sa_run(ins, chains, 0, seed=77, t0_samples=300, lanes=lanes)
    torch.cuda.synchronize()
    pen, perm, gid = lib.best_get(ins)
    pr = oracle.Problem.from_instance(inst)
    T0 = oracle.t0(pr, oracle.CDD, 77, 300)
    assert float(res["T0"].item()) == T0
    ref = oracle.sa_run(pr, oracle.sa_params(chains=chains, steps=0, seed=77), T0)
    assert (pen, gid) == (ref["E_best"], ref["g"])
    assert np.array_equal(perm, ref["best"])


@pytest.mark.parametrize("n", [1, 2, 3])
@pytest.mark.parametrize("problem", ["cdd", "ucddcp"])
def test_tiny_n_sa_and_dpso(lib, n, problem):
    # degenerate sizes: Pert = min(4, n) slots, swaps/crossovers on 1-3 positions
    import torch

    inst = gen.ucddcp_instance(n, 3) if problem == "ucddcp" else gen.cdd_instance(n, 3, 0.4)
    ins = lib.Instance.from_gen(inst)
    pr = oracle.Problem.from_instance(inst)
    P = oracle.UCDDCP if problem == "ucddcp" else oracle.CDD
    res = lib.sa_run(ins, 33, 60, problem=problem, seed=5, t0_samples=100, trace=True)
    torch.cuda.synchronize()
    pen, perm, gid = lib.best_get(ins)
    T0 = oracle.t0(pr, P, 5, 100)
    p = oracle.sa_params(problem=P, chains=33, steps=60, seed=5)
    tr = res["trace"].cpu().numpy()
    for c in range(33):
        ref = oracle.sa_chain(pr, p, T0, c, trace=True)
        assert np.array_equal(tr[c] >> 1, ref["E_new"]), c
        assert np.array_equal((tr[c] & 1).astype(bool), ref["accepted"]), c
    ref = oracle.sa_run(pr, p, T0)
    assert (pen, gid) == (ref["E_best"], ref["g"]) and np.array_equal(perm, ref["best"])
    if n == 1:  # F1-F3 need two positions: the ABI refuses (include/cdd.h, dpso_run)
        with pytest.raises(lib.CddError) as e:
            lib.dpso_run(ins, 20, 7, problem=problem, seed=6)
        assert e.value.code == lib.CDD_EINVAL
        return
    r2 = lib.dpso_run(ins, 20, 7, problem=problem, seed=6, trace=True)
    torch.cuda.synchronize()
    pen, perm, gid = lib.best_get(ins)
    ref = oracle.dpso_run(pr, oracle.dpso_params(problem=P, particles=20, iters=7, seed=6), trace=True)
    assert np.array_equal(r2["gbest_trace"].cpu().numpy()[:7], ref["gbest_trace"])
    assert (pen, gid) == (ref["E_best"], ref["id"]) and np.array_equal(perm, ref["best"])


def test_dpso_zero_iterations(lib):
    import torch

    inst = gen.cdd_instance(300, 4, 0.2)
    ins = lib.Instance.from_gen(inst)
    lib.dpso_run(ins, 100, 0, seed=12)
    torch.cuda.synchronize()
    pen, perm, gid = lib.best_get(ins)
    pr = oracle.Problem.from_instance(inst)
    ref = oracle.dpso_run(pr, oracle.dpso_params(particles=100, iters=0, seed=12))
    assert (pen, gid) == (ref["E_best"], ref["id"]) and np.array_equal(perm, ref["best"])


def test_maximum_n_sa_and_dpso(lib):
    # n = 1024 is the largest size the group layouts hold (8 lanes x 128 positions)
    import torch

    inst = gen.cdd_instance(1024, 5, 0.4)
    ins = lib.Instance.from_gen(inst)
    pr = oracle.Problem.from_instance(inst)
    lib.sa_run(ins, 40, 30, seed=9, t0_samples=200)
    torch.cuda.synchronize()
    pen, perm, gid = lib.best_get(ins)
    T0 = oracle.t0(pr, oracle.CDD, 9, 200)
    ref = oracle.sa_run(pr, oracle.sa_params(chains=40, steps=30, seed=9), T0)
    assert (pen, gid) == (ref["E_best"], ref["g"]) and np.array_equal(perm, ref["best"])
    lib.dpso_run(ins, 24, 4, seed=10)
    torch.cuda.synchronize()
    pen, perm, gid = lib.best_get(ins)
    ref = oracle.dpso_run(pr, oracle.dpso_params(particles=24, iters=4, seed=10))
    assert (pen, gid) == (ref["E_best"], ref["id"]) and np.array_equal(perm, ref["best"])


def test_run_argument_errors(lib):
    inst = gen.cdd_instance(20, 1, 0.4)
    ins = lib.Instance.from_gen(inst)
    for call in (lambda: lib.sa_run(ins, 0, 10),
                 lambda: lib.dpso_run(ins, 0, 10),
                 lambda: lib.sa_run(ins, 8, 10, problem="ucddcp")):  # CDD-only instance (no M, gamma)
        with pytest.raises(lib.CddError) as e:
            call()
        assert e.value.code == lib.CDD_EINVAL
