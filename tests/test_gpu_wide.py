"""GPU parity of the generic ("wide") path: instances outside the packed record ranges (P:29-49
define P, alpha, beta, gamma, d as general non-negative integers) -- n up to 32767, large values,
int64 penalties -- against the oracle, element by element."""
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


def _data(n, seed, pmax=1000, wmax=10_000, zero=False):
    rng = np.random.default_rng(seed)
    lo = 0 if zero else 1
    P = rng.integers(1, pmax + 1, n).astype(np.int32)
    a = rng.integers(lo, wmax + 1, n).astype(np.int32)
    b = rng.integers(lo, wmax + 1, n).astype(np.int32)
    M = (P - rng.integers(0, P)).astype(np.int32)
    g = rng.integers(lo, wmax + 1, n).astype(np.int32)
    return P, a, b, M, g


def _perms(batch, n, seed, ld=None):
    return gen.random_perms(batch, n, seed, ld)


def _dev(x):
    import torch

    return torch.from_numpy(np.ascontiguousarray(x)).cuda()


def test_verdict_example_evaluates(lib):
    # Instance([1000]*10, [1000]*10, [1]*10, ...) must evaluate instead of raising
    P = [1000] * 10
    ins = lib.Instance(P, [1000] * 10, [1] * 10, 4000)
    assert ins.wide and ins.query()["generic"]
    perms = _perms(64, 10, 1)
    z = lib.cdd_eval_batch(ins, _dev(perms)).cpu().numpy()
    pr = oracle.Problem(P, [1000] * 10, [1] * 10, 4000)
    assert np.array_equal(z, oracle.eval_batch(pr, perms))


@pytest.mark.parametrize("n", [7, 300, 1025, 2048, 2049, 4096])
@pytest.mark.parametrize("h", [0.0, 0.2, 0.6, 1.0, 1.7])
def test_cdd_wide_parity(lib, n, h):
    P, a, b, M, g = _data(n, n * 7 + int(h * 10))
    d = int(h * int(P.sum()))
    ins = lib.Instance(P, a, b, d)
    assert ins.wide
    batch = 64 if n <= 2048 else 24
    perms = _perms(batch, n, n + 1, ld=n + 3)  # odd stride
    z = lib.cdd_eval_batch(ins, _dev(perms)).cpu().numpy()
    want = oracle.eval_batch(oracle.Problem(P, a, b, d), perms)
    assert np.array_equal(z, want)
    if n >= 300:
        assert z.max() > 2**32  # beyond the packed key's 32 bits


@pytest.mark.parametrize("n", [9, 500, 2100])
def test_ucddcp_wide_parity(lib, n):
    P, a, b, M, g = _data(n, 100 + n)
    d = int(P.sum()) + 5
    ins = lib.Instance(P, a, b, d, M, g)
    perms = _perms(32 if n < 2000 else 8, n, 3 + n)
    z = lib.ucddcp_eval_batch(ins, _dev(perms)).cpu().numpy()
    want = oracle.eval_batch(oracle.Problem(P, a, b, d, M, g), perms, oracle.UCDDCP)
    assert np.array_equal(z, want)


def test_wide_zero_weights_and_edges(lib):
    # zero penalties (flat optima), d = 0, d >= sum P, n = 1 and 2
    for n, seed in [(1, 1), (2, 2), (40, 3), (1500, 4)]:
        P, a, b, M, g = _data(n, seed, zero=True)
        for d in [0, int(P.sum()) // 3, int(P.sum()), int(P.sum()) + 1000]:
            ins = lib.Instance(P, a, b, d, M, g)
            perms = _perms(16, n, seed + d)
            z = lib.cdd_eval_batch(ins, _dev(perms)).cpu().numpy()
            assert np.array_equal(z, oracle.eval_batch(oracle.Problem(P, a, b, d), perms)), (n, d)
            if d >= P.sum():
                zu = lib.ucddcp_eval_batch(ins, _dev(perms)).cpu().numpy()
                assert np.array_equal(zu, oracle.eval_batch(oracle.Problem(P, a, b, d, M, g), perms,
                                                            oracle.UCDDCP)), (n, d)


def test_wide_max_n_sampled(lib):
    # n = 32767 (int16 ids): a CTA per sequence; sampled rows through the oracle
    n = 32767
    P, a, b, M, g = _data(n, 9, pmax=50, wmax=60)
    d = int(0.4 * int(P.sum()))
    ins = lib.Instance(P, a, b, d, M, g)
    perms = _perms(6, n, 11)
    z = lib.cdd_eval_batch(ins, _dev(perms)).cpu().numpy()
    assert np.array_equal(z, oracle.eval_batch(oracle.Problem(P, a, b, d), perms))
    dU = int(P.sum())
    insU = lib.Instance(P, a, b, dU, M, g)
    zu = lib.ucddcp_eval_batch(insU, _dev(perms[:2])).cpu().numpy()
    assert np.array_equal(zu, oracle.eval_batch(oracle.Problem(P, a, b, dU, M, g), perms[:2], oracle.UCDDCP))


def test_wide_bad_ids_flag(lib):
    n = 3000
    P, a, b, M, g = _data(n, 5)
    ins = lib.Instance(P, a, b, 1000)
    perms = _perms(4, n, 2)
    perms[2, 17] = n + 5
    lib.cdd_eval_batch(ins, _dev(perms))
    with pytest.raises(lib.CddError) as e:
        lib.cdd_check(ins)
    assert e.value.code == lib.CDD_EDATA
    lib.cdd_check(ins)  # cleared


def test_wide_erange_and_best_ptrs(lib):
    big = [2**31 - 1] * 4
    with pytest.raises(lib.CddError) as e:
        lib.Instance(big, big, big, 10)
    assert e.value.code == lib.CDD_ERANGE


@pytest.mark.parametrize("problem", ["cdd", "ucddcp"])
def test_wide_schedules(lib, problem):
    n = 1200
    P, a, b, M, g = _data(n, 31)
    d = int(P.sum()) + 7 if problem == "ucddcp" else int(0.5 * int(P.sum()))
    ins = lib.Instance(P, a, b, d, M, g)
    perms = _perms(12, n, 4)
    out = lib.cdd_schedule_batch(ins, _dev(perms), problem)
    C = out["C"].cpu().numpy()
    pen = out["penalty"].cpu().numpy()
    st = out["start"].cpu().numpy()
    X = out["X"].cpu().numpy() if problem == "ucddcp" else np.zeros_like(C, dtype=np.int32)
    pr = oracle.Problem(P, a, b, d, M, g)
    for r in range(len(perms)):
        J = perms[r, :n].astype(np.int64)
        z = oracle.ucddcp_eval(pr, J) if problem == "ucddcp" else oracle.cdd_eval(pr, J)
        assert pen[r] == z
        # a valid schedule: no idle time, start >= 0, compressions in {0, P - M}, eq. (1)/(2) = pen
        p_eff = P[J].astype(np.int64) - X[r]
        assert st[r] >= 0 and np.array_equal(C[r], st[r] + np.cumsum(p_eff))
        assert np.all((X[r] == 0) | (X[r] == P[J] - M[J]))
        Zs = (a[J] * np.maximum(0, d - C[r]) + b[J] * np.maximum(0, C[r] - d)).sum() + (g[J] * X[r]).sum()
        assert Zs == z


def _sa_both(lib, P, a, b, d, M, g, problem, chains, steps, seed, move="pert_fy", T0=0.0, samples=300,
             mu=0.88):
    import torch

    ins = lib.Instance(P, a, b, d, M, g)
    assert ins.wide
    res = lib.sa_run(ins, chains, steps, problem=problem, seed=seed, move=move, T0=T0, t0_samples=samples,
                     trace=True, chain_best=True, chain_final=True, mu=mu)
    torch.cuda.synchronize()
    pr = oracle.Problem(P, a, b, d, M, g)
    PP = oracle.CDD if problem == "cdd" else oracle.UCDDCP
    T0r = T0 if T0 > 0 else oracle.t0(pr, PP, seed, samples)
    assert float(res["T0"].item()) == T0r
    mv = {"pert_fy": oracle.MOVE_PERT_FY, "swap": oracle.MOVE_SWAP, "insert": oracle.MOVE_INSERT,
          "window": oracle.MOVE_WINDOW}[move]
    p = oracle.sa_params(problem=PP, chains=chains, steps=steps, seed=seed, move=mv, mu=mu)
    tr = res["trace"].cpu().numpy()
    cb = res["chain_best"].cpu().numpy()
    cf = res["chain_final"].cpu().numpy()
    for c in range(chains):
        ref = oracle.sa_chain(pr, p, T0r, c, trace=True)
        assert np.array_equal(tr[c] >> 1, ref["E_new"]), c
        assert np.array_equal((tr[c] & 1).astype(bool), ref["accepted"]), c
        assert cb[c] == ref["E_best"] and cf[c] == ref["E_final"], c
    full = oracle.sa_run(pr, p, T0r)
    pen, perm, gid = lib.best_get(ins)
    assert (pen, gid) == (full["E_best"], full["g"]) and np.array_equal(perm, full["best"])
    return ins


@pytest.mark.parametrize("move", ["pert_fy", "swap", "insert", "window"])
def test_wide_sa_parity(lib, move):
    P, a, b, M, g = _data(60, 77, wmax=100_000)
    ins = _sa_both(lib, P, a, b, int(0.4 * int(P.sum())), M, g, "cdd", 24, 300, 5, move=move)
    with pytest.raises(lib.CddError):
        lib.best_device_ptrs(ins)  # the packed key cannot hold these penalties
    pen_id, perm = lib.best_device_tensors_wide(ins)
    assert int(pen_id[0].item()) == lib.best_get(ins)[0] > 2**32


def test_wide_sa_ucddcp_and_long(lib):
    P, a, b, M, g = _data(40, 78)
    _sa_both(lib, P, a, b, int(P.sum()), M, g, "ucddcp", 16, 200, 6, move="insert", mu=1.0, T0=1e7)
    P, a, b, M, g = _data(1500, 79, pmax=200, wmax=300)
    _sa_both(lib, P, a, b, int(0.6 * int(P.sum())), M, g, "cdd", 6, 60, 7, mu=1.0, T0=5e6)


def test_wide_t0(lib):
    P, a, b, M, g = _data(3000, 80)
    d = int(0.3 * int(P.sum()))
    ins = lib.Instance(P, a, b, d, M, g)
    t = float(lib.sa_t0(ins, "cdd", seed=4, samples=700).item())
    assert t == oracle.t0(oracle.Problem(P, a, b, d, M, g), oracle.CDD, 4, 700)


def test_wide_other_entry_points_refuse(lib):
    P, a, b, M, g = _data(30, 81)
    ins = lib.Instance(P, a, b, 100, M, g)
    with pytest.raises(lib.CddError):
        lib.dpso_run(ins, 64, 5)
    with pytest.raises(lib.CddError):
        lib.sa_sync_run(ins, 64, 5, 3)
    with pytest.raises(lib.CddError):
        lib.sa_run(ins, 64, 5, lanes=8)
