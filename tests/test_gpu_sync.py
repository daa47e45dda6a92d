"""GPU parity of synchronous SA against oracle.sa_sync: per-level
minimum final penalties, the best-ever penalty / chain / sequence, bit for bit."""
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


MOVES = {"pert_fy": oracle.MOVE_PERT_FY, "insert": oracle.MOVE_INSERT,
         "window": oracle.MOVE_WINDOW, "swap": oracle.MOVE_SWAP}


def _both(lib, inst, problem, chains, M, levels, seed, lanes=0, T0=0.0, samples=400, mu=0.88,
          move="pert_fy"):
    import torch

    ins = lib.Instance.from_gen(inst)
    ss = lib.sa_sync_run(ins, chains, M, levels, problem=problem, seed=seed, lanes=lanes, T0=T0,
                         t0_samples=samples, mu=mu, move=move)
    torch.cuda.synchronize()
    pen, perm, gid = lib.best_get(ins)
    pr = oracle.Problem.from_instance(inst)
    P = oracle.CDD if problem == "cdd" else oracle.UCDDCP
    T0_ref = T0 if T0 > 0 else oracle.t0(pr, P, seed, samples)
    assert float(ss.T0.item()) == T0_ref
    p = oracle.sa_params(problem=P, chains=chains, steps=M, mu=mu, seed=seed, move=MOVES[move])
    ref = oracle.sa_sync(pr, p, T0_ref, levels)
    return ss, (pen, perm, gid), ref


@pytest.mark.parametrize("lanes", [0, 16, 8, 4])
@pytest.mark.parametrize("problem,n,chains,M,levels", [("cdd", 40, 64, 30, 12),
                                                       ("cdd", 300, 48, 20, 6),
                                                       ("ucddcp", 100, 40, 25, 8),
                                                       ("cdd", 1000, 24, 10, 4)])
def test_sync_sa_parity(lib, problem, n, chains, M, levels, lanes):
    if lanes == 4 and n > 256:
        pytest.skip("lanes=4 needs n <= 256")
    inst = gen.ucddcp_instance(n, 3) if problem == "ucddcp" else gen.cdd_instance(n, 3, 0.4)
    ss, (pen, perm, gid), ref = _both(lib, inst, problem, chains, M, levels, seed=11 + n,
                                      lanes=lanes)
    assert np.array_equal(ss.level_min.cpu().numpy(), ref["level_min_E"])
    assert (pen, gid) == (ref["E_best"], ref["g"])
    assert np.array_equal(perm, ref["best"])


@pytest.mark.parametrize("move", ["insert", "window"])
@pytest.mark.parametrize("problem,n,lanes", [("cdd", 200, 8), ("ucddcp", 90, 4), ("cdd", 1000, 8)])
def test_sync_sa_other_moves(lib, move, problem, n, lanes):
    inst = gen.ucddcp_instance(n, 5) if problem == "ucddcp" else gen.cdd_instance(n, 5, 0.4)
    ss, (pen, perm, gid), ref = _both(lib, inst, problem, 32, 15, 6, seed=3 + n, lanes=lanes,
                                      move=move)
    assert np.array_equal(ss.level_min.cpu().numpy(), ref["level_min_E"])
    assert (pen, gid) == (ref["E_best"], ref["g"]) and np.array_equal(perm, ref["best"])


def test_sync_sa_greedy_and_constant_temperature(lib):
    inst = gen.cdd_instance(64, 2, 0.6)
    ss, (pen, perm, gid), ref = _both(lib, inst, "cdd", 32, 15, 10, seed=4, T0=1e-9)
    lm = ss.level_min.cpu().numpy()
    assert np.array_equal(lm, ref["level_min_E"]) and np.all(np.diff(lm) <= 0)
    ss, (pen, perm, gid), ref = _both(lib, inst, "cdd", 32, 15, 10, seed=4, T0=300.0, mu=1.0)
    assert np.array_equal(ss.level_min.cpu().numpy(), ref["level_min_E"]) and pen == ref["E_best"]


def test_sync_sa_emulated_two_ranks(lib):
    # two "ranks" on one GPU: chain ids [0, C) and [C, 2C), s^min exchanged between levels (what
    # dist.sa_sync_run_distributed does with NCCL) == one run of 2C chains
    import torch

    inst = gen.cdd_instance(120, 5, 0.4)
    C, M, L, seed = 40, 12, 7, 21
    ranks = [lib.Instance.from_gen(inst) for _ in range(2)]
    ss = [lib.SaSync(ranks[r], C, M, L, seed=seed, chain_offset=r * C, t0_samples=300) for r in range(2)]
    for j in range(L):
        for s in ss:
            s.level(j)
        ex = [s.exchange_tensors() for s in ss]
        keys = [int(k.item()) for k, _ in ex]
        w = int(np.argmin(keys))
        for r in range(2):
            ex[r][0].fill_(keys[w])
            ex[r][1].copy_(ex[w][1])
    torch.cuda.synchronize()
    bests = [lib.best_get(r) for r in ranks]
    one = lib.Instance.from_gen(inst)
    lib.sa_sync_run(one, 2 * C, M, L, seed=seed, t0_samples=300)
    pen, perm, gid = lib.best_get(one)
    assert min(b[0] for b in bests) == pen


def test_sync_sa_argument_checks(lib):
    ins = lib.Instance.from_gen(gen.cdd_instance(50, 1, 0.4))
    with pytest.raises(lib.CddError):
        lib.sa_sync_run(ins, 64, 10, 3, lanes=32, T0=5.0)
    with pytest.raises(lib.CddError):
        lib.sa_sync_run(ins, 64, 0, 3, T0=5.0)
    heavy = lib.Instance.from_gen(gen.ranged_instance(80, 3, p=(1, 3), alpha=(200, 400),
                                                      beta=(1, 5), h=0.5))
    with pytest.raises(lib.CddError):
        lib.sa_sync_run(heavy, 64, 10, 3, T0=5.0)
