"""GPU parity of cdd_schedule_batch: the optimal schedule of a sequence.

The penalty is unique and compared with the oracle element by element; the schedule itself is
unique unless the cost has a flat optimum (some prefix S_k of alpha + beta equals sum beta), so
it is compared with the oracle's on instances without such a tie and otherwise checked for
validity (no idle time, start >= 0, its eq. (1)/(2) cost equals the penalty)."""
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


def _tie(inst, perm):
    ab = (inst.alpha + inst.beta)[perm]
    S = np.concatenate([[0], np.cumsum(ab)[:-1]])
    return bool(np.any(S == int(inst.beta.sum())))


def _cost(inst, perm, C, X, d):
    a, b = inst.alpha[perm].astype(np.int64), inst.beta[perm].astype(np.int64)
    z = np.sum(a * np.maximum(0, d - C) + b * np.maximum(0, C - d))
    if X is not None:
        z += np.sum(inst.gamma[perm].astype(np.int64) * X)
    return int(z)


CASES = [("cdd", 1, 0.4), ("cdd", 5, 0.0), ("cdd", 37, 0.2), ("cdd", 100, 0.6), ("cdd", 333, 1.3),
         ("cdd", 1000, 0.4), ("ucddcp", 7, None), ("ucddcp", 200, None), ("ucddcp", 1000, None)]


@pytest.mark.parametrize("problem,n,h", CASES)
def test_schedule_matches_oracle(lib, problem, n, h):
    import torch

    inst = gen.ucddcp_instance(n, 5) if problem == "ucddcp" else gen.cdd_instance(n, 5, h)
    ins = lib.Instance.from_gen(inst)
    B = 48
    perms = gen.random_perms(B, n, seed=17 + n)
    ld = perms.shape[1]
    out = lib.cdd_schedule_batch(ins, torch.from_numpy(perms).cuda(), problem)
    torch.cuda.synchronize()
    C, pen, start = out["C"].cpu().numpy(), out["penalty"].cpu().numpy(), out["start"].cpu().numpy()
    X = out["X"].cpu().numpy() if "X" in out else None
    pr = oracle.Problem.from_instance(inst)
    P = inst.P.astype(np.int64)
    for r in range(B):
        perm = perms[r, :n].astype(np.int64)
        if problem == "cdd":
            z_ref, w = oracle.cdd_eval(pr, perms[r, :n], walk=True)
            C_ref, X_ref, p_eff = w["C"], None, P[perm]
        else:
            z_ref, X_ref, C_ref = oracle.ucddcp_eval(pr, perms[r, :n], detail=True)
            p_eff = P[perm] - X[r]
        assert pen[r] == z_ref, r
        # validity: no idle time, non-negative start, cost of the schedule = penalty
        assert start[r] >= 0 and C[r, 0] - p_eff[0] == start[r], r
        assert np.array_equal(np.diff(C[r]), p_eff[1:]), r
        assert _cost(inst, perm, C[r], None if X is None else X[r], inst.d) == pen[r], r
        if not _tie(inst, perm):
            assert np.array_equal(C[r], C_ref), r
            if X is not None:
                assert np.array_equal(X[r], X_ref), r
    lib.cdd_check(ins)  # raises if any id was out of range
    assert ld >= n


def test_schedule_of_sa_best(lib):
    inst = gen.cdd_instance(200, 2, 0.4)
    ins = lib.Instance.from_gen(inst)
    lib.sa_run(ins, 2048, 300, seed=3, t0_samples=500)
    pen, perm, gid = lib.best_get(ins)
    C, X, start, z = lib.schedule_get(ins, perm)
    assert z == pen and X is None
    assert _cost(inst, perm.astype(np.int64), C, None, inst.d) == pen


def test_schedule_table1_example(lib):
    # Table I, CDD d=16: optimum 81 with the sequence in id order, shift 5
    inst = gen.table1()
    ins = lib.Instance.from_gen(inst)
    C, X, start, z = lib.schedule_get(ins, np.arange(5, dtype=np.int16))
    assert z == 81
    golden = oracle.cdd_eval(oracle.Problem.from_instance(inst), np.arange(5, dtype=np.int16), walk=True)[1]
    assert start == golden["s"] and np.array_equal(C, golden["C"])


@pytest.mark.parametrize("n,pad", [(257, 7), (333, 3), (512, 0), (999, 9), (1000, 8), (1001, 7)])
def test_schedule_vector_path_padding_and_bad_ids(lib, n, pad):
    # n > 256 stages the ids by 16-byte chunks loaded one row ahead: garbage in the caller's padding
    # past n is ignored, odd n stores C one position at a time, out-of-range ids raise the flag
    import torch

    inst = gen.cdd_instance(n, 9, 0.4)
    ins = lib.Instance.from_gen(inst)
    perms = gen.random_perms(70, n, seed=n + pad, ld=gen.pad_ld(n) + (8 if pad else 0))
    perms[:, n:] = 4321
    out = lib.cdd_schedule_batch(ins, torch.from_numpy(perms).cuda())
    pen = out["penalty"].cpu().numpy()
    C = out["C"].cpu().numpy()
    assert np.array_equal(pen, _oracle_pens(inst, perms, n))
    P = inst.P.astype(np.int64)
    for r in range(0, 70, 7):
        perm = perms[r, :n].astype(np.int64)
        assert np.array_equal(np.diff(C[r]), P[perm][1:]), r
        assert _cost(inst, perm, C[r], None, inst.d) == pen[r], r
    lib.cdd_check(ins)
    q = perms.copy()
    q[69, n - 1] = n  # last row, last position (the straddling chunk when n % 8 != 0)
    lib.cdd_schedule_batch(ins, torch.from_numpy(q).cuda())
    with pytest.raises(lib.CddError):
        lib.cdd_check(ins)


def _oracle_pens(inst, perms, n):
    pr = oracle.Problem.from_instance(inst)
    return oracle.eval_batch_threaded(pr, perms, oracle.CDD)
