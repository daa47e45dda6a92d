"""Pins of the oracle's sequence evaluators (CPU only).

Each test ties or_cdd_eval / or_ucddcp_eval to something other than itself: the paper's worked
example (Table I), exhaustive solvers of the fixed-sequence LP, the theorems and
properties the paper states, and the V-shape property.
"""
import json
import os

import numpy as np
import pytest

import gen
import oracle
from tests import bruteforce as bf

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "table1.json")))


def _prob(inst, d=None):
    return oracle.Problem.from_instance(inst, d=d)


# ----------------------------------------------------------------------------- Table I (CDD)
def test_table1_cdd_walk_every_intermediate_value():
    g = GOLD["cdd"]
    t = gen.table1()
    pr = _prob(t, d=g["d"])
    J = np.array(GOLD["sequence"])
    Z, w = oracle.cdd_eval(pr, J, walk=True)
    C0 = np.cumsum(t.P[J])
    assert list(C0) == g["C_initial"]
    assert list(C0 - g["d"]) == g["DT_initial"]
    assert w["tau"] == g["tau"]
    assert (w["pe0"], w["pl0"]) == (g["pe0"], g["pl0"])
    assert w["first_shift"] == g["first_shift"]
    assert list(C0 + w["first_shift"] - g["d"]) == g["DT_after_first_shift"]
    assert (w["pe"][0], w["pl"][0]) == (g["pe1"], g["pl1"])
    assert w["s"] == g["first_shift"] + g["second_shift"]
    assert w["r"] == g["final_job_at_d"]
    assert w["C"][w["r"] - 1] == g["d"]
    assert Z == g["penalty"]


def test_table1_ucddcp():
    g = GOLD["ucddcp"]
    t = gen.table1()
    pr = _prob(t, d=g["d"])
    J = np.array(GOLD["sequence"])
    Z, X, C = oracle.ucddcp_eval(pr, J, detail=True)
    assert Z == g["penalty"]
    assert list(X) == g["X"]
    assert C[g["job_at_d"] - 1] == g["d"]
    # the two printed gains: compressing job 5 alone, then job 4
    Zcdd = oracle.cdd_eval(pr, J)
    assert Zcdd == GOLD["cdd"]["penalty"]  # translation invariant for d >= sum P (T8)
    assert Zcdd - Z == g["gain_job5"] + g["gain_job4"]


def test_table1_ucddcp_requires_unrestricted_d():
    pr = _prob(gen.table1(), d=20)  # sum P = 21
    with pytest.raises(ValueError):
        oracle.ucddcp_eval(pr, np.arange(5))


# ----------------------------------------------------------------------- brute-force pins
def _small_cases(count, nmax, seed0=0, **kw):
    rng = np.random.default_rng(1234 + seed0)
    for c in range(count):
        n = int(rng.integers(1, nmax + 1))
        inst = gen.random_small(n, seed0 * 100000 + c, **kw)
        J = rng.permutation(n)
        yield inst, J


@pytest.mark.parametrize("zero_weights", [False, True])
def test_cdd_walk_equals_shift_bruteforce(zero_weights):
    for inst, J in _small_cases(1500, 8, seed0=1 + zero_weights, zero_weights=zero_weights):
        pr = _prob(inst)
        assert oracle.cdd_eval(pr, J) == bf.shift_bf(inst.P, inst.alpha, inst.beta, inst.d, J)


def test_cdd_walk_equals_idle_allowed_dp():
    # DP over integer completion times with idle time allowed: pins the no-idle property [9]
    for inst, J in _small_cases(300, 6, seed0=3):
        pr = _prob(inst)
        assert oracle.cdd_eval(pr, J) == bf.dp_schedule(inst.P, inst.alpha, inst.beta, inst.d, J)


def test_cdd_walk_equals_lp_solver():
    # the LP of P:65-69 for fixed delta (continuous variables) solved by scipy HiGHS
    for inst, J in _small_cases(120, 7, seed0=4):
        pr = _prob(inst)
        lp = bf.lp_schedule(inst.P, inst.alpha, inst.beta, inst.d, J)
        assert abs(oracle.cdd_eval(pr, J) - lp) < 1e-6


def test_cdd_generated_instances_vs_shift_bruteforce():
    # generator-range instances (p<=20, alpha<=10, beta<=15), all four h, n up to 40
    rng = np.random.default_rng(7)
    for k in range(1, 6):
        for h in gen.H_VALUES:
            inst = gen.cdd_instance(40, k, h)
            pr = _prob(inst)
            for _ in range(5):
                J = rng.permutation(40)
                assert oracle.cdd_eval(pr, J) == bf.shift_bf(inst.P, inst.alpha, inst.beta, inst.d, J)


def test_cdd_unrestricted_invariance():
    # T8: for d >= sum P the penalty does not depend on d (translation of the schedule)
    for inst, J in _small_cases(400, 8, seed0=5):
        s = int(inst.P.sum())
        Z1 = oracle.cdd_eval(_prob(inst, d=s), J)
        Z2 = oracle.cdd_eval(_prob(inst, d=s + 17), J)
        assert Z1 == Z2


def test_theorem1_holds_at_the_walks_schedule():
    # Theorem 1.  Case 2 (C_r = d) at the final schedule; in the start-0 case the
    # due date lies inside job r = tau+1 and Case 1 (i) holds for k = 1..min(tau+1, n).
    for inst, J in _small_cases(1500, 9, seed0=6):
        pr = _prob(inst)
        Z, w = oracle.cdd_eval(pr, J, walk=True)
        a = inst.alpha[J].astype(np.int64)
        b = inst.beta[J].astype(np.int64)
        n = len(J)
        A = lambda lo, hi: int(a[lo - 1:hi].sum())  # sum_{i=lo}^{hi} alpha_i (1-based)
        B = lambda lo, hi: int(b[lo - 1:hi].sum())
        r = w["r"]
        if r >= 1:
            assert w["C"][r - 1] == inst.d
            for k in range(r, n + 1):
                assert B(k + 1, n) <= A(1, k)          # Case 2 (i)
            for k in range(1, r + 1):
                assert A(1, k - 1) <= B(k, n)          # Case 2 (ii)
        else:
            assert w["s"] == 0
            for k in range(1, min(w["tau"] + 1, n) + 1):
                assert A(1, k - 1) <= B(k, n)          # Case 1 (i)


def test_v_shape_min_over_all_sequences():
    # min over n! sequences == min over V-shaped sequences (there is a V-shaped optimum)
    for c in range(60):
        n = 3 + c % 4
        inst = gen.random_small(n, 777 + c)
        pr = _prob(inst)
        allZ = {tuple(J): oracle.cdd_eval(pr, np.array(J)) for J in bf.all_sequences(n)}
        zmin = min(allZ.values())
        vmin = min(z for J, z in allZ.items() if bf.v_shaped(inst.P, inst.alpha, inst.beta, list(J)))
        assert zmin == vmin


def test_nfact_optimum_matches_dp_optimum():
    # the best sequence found by enumerating n! and evaluating with the walk is the global optimum
    # of the fixed-sequence DP minimised over sequences (n <= 5)
    for c in range(15):
        n = 2 + c % 4
        inst = gen.random_small(n, 4242 + c)
        pr = _prob(inst)
        seqs = bf.all_sequences(n)
        z_walk = min(oracle.cdd_eval(pr, np.array(J)) for J in seqs)
        z_dp = min(bf.dp_schedule(inst.P, inst.alpha, inst.beta, inst.d, J) for J in seqs)
        assert z_walk == z_dp


# ------------------------------------------------------------------------------- UCDDCP
def test_ucddcp_equals_integer_dp_with_compression():
    for inst, J in _small_cases(250, 5, seed0=8):
        d = int(inst.P.sum()) + (inst.seed % 3)
        pr = _prob(inst, d=d)
        z = oracle.ucddcp_eval(pr, J)
        assert z == bf.dp_schedule(inst.P, inst.alpha, inst.beta, d, J, M=inst.M, g=inst.gamma)


def test_ucddcp_equals_lp_solver():
    for inst, J in _small_cases(120, 7, seed0=9):
        d = int(inst.P.sum())
        pr = _prob(inst, d=d)
        lp = bf.lp_schedule(inst.P, inst.alpha, inst.beta, d, J, M=inst.M, g=inst.gamma)
        assert abs(oracle.ucddcp_eval(pr, J) - lp) < 1e-6


def test_ucddcp_properties_1_and_2():
    for inst, J in _small_cases(600, 9, seed0=10):
        d = int(inst.P.sum())
        pr = _prob(inst, d=d)
        Z, X, C = oracle.ucddcp_eval(pr, J, detail=True)
        _, w = oracle.cdd_eval(pr, J, walk=True)
        # Property 1: the due-date position of the CDD optimum is kept
        assert C[w["r"] - 1] == d
        # Property 2: compress to the minimum or not at all
        full = inst.P[J] - inst.M[J]
        assert all(x == 0 or x == f for x, f in zip(X, full))
        assert Z <= oracle.cdd_eval(pr, J)


def test_ucddcp_generated_instances_vs_dp():
    rng = np.random.default_rng(11)
    for k in range(1, 4):
        inst = gen.ucddcp_instance(7, k)
        pr = _prob(inst)
        for _ in range(4):
            J = rng.permutation(7)
            assert oracle.ucddcp_eval(pr, J) == bf.dp_schedule(
                inst.P, inst.alpha, inst.beta, inst.d, J, M=inst.M, g=inst.gamma)


def test_eval_batch_matches_single():
    inst = gen.cdd_instance(50, 3, 0.4)
    pr = _prob(inst)
    perms = gen.random_perms(64, 50, 5)
    out = oracle.eval_batch(pr, perms)
    assert list(out) == [oracle.cdd_eval(pr, r[:50]) for r in perms]
    outt = oracle.eval_batch_threaded(pr, perms, threads=3)
    assert list(outt) == list(out)


# ------------------------------------------------- wide value ranges (the generic path, §8(b))
def _wide_cases(count, nmax, seed, pmax, wmax, rng_h=True):
    rng = np.random.default_rng(seed)
    for c in range(count):
        n = int(rng.integers(1, nmax + 1))
        P = rng.integers(1, pmax + 1, n).astype(np.int64)
        a = rng.integers(0, wmax + 1, n).astype(np.int64)
        b = rng.integers(0, wmax + 1, n).astype(np.int64)
        M = (P - rng.integers(0, P)).astype(np.int64)           # 1 <= M <= P
        g = rng.integers(0, wmax + 1, n).astype(np.int64)
        h = float(rng.choice([0.0, 0.2, 0.4, 0.6, 0.8, 1.0, 1.3])) if rng_h else 1.0
        d = int(h * int(P.sum()))
        yield P, a, b, M, g, d, rng.permutation(n)


def test_cdd_wide_values_vs_breakpoint_bruteforce():
    # P:29-59 define P, alpha, beta, d as general non-negative integers: p <= 1000,
    # alpha, beta <= 10^4, and n up to 300 (exact big-integer brute force over starts)
    for P, a, b, M, g, d, J in _wide_cases(300, 12, 21, 1000, 10_000):
        pr = oracle.Problem(P, a, b, d)
        assert oracle.cdd_eval(pr, J) == bf.breakpoint_bf(P, a, b, d, J)
    for P, a, b, M, g, d, J in _wide_cases(12, 300, 22, 1000, 10_000):
        pr = oracle.Problem(P, a, b, d)
        assert oracle.cdd_eval(pr, J) == bf.breakpoint_bf(P, a, b, d, J)


def test_cdd_huge_values_int64_exact():
    # penalties far beyond 2^32: int32 data at the top of its range, exact in int64
    for P, a, b, M, g, d, J in _wide_cases(60, 9, 23, 2_000_000, 200_000_000):
        pr = oracle.Problem(P, a, b, d)
        z = bf.breakpoint_bf(P, a, b, d, J)
        assert z < 2**63 and oracle.cdd_eval(pr, J) == z
    # shift brute force on moderate values agrees with the breakpoint enumeration (pins the helper)
    for P, a, b, M, g, d, J in _wide_cases(100, 6, 24, 30, 50):
        assert bf.breakpoint_bf(P, a, b, d, J) == bf.shift_bf(P, a, b, d, J)


def test_ucddcp_wide_values_vs_vertex_bruteforce():
    for P, a, b, M, g, d, J in _wide_cases(150, 8, 25, 1000, 10_000, rng_h=False):
        d = int(P.sum()) + int(P[0])
        pr = oracle.Problem(P, a, b, d, M, g)
        assert oracle.ucddcp_eval(pr, J) == bf.ucddcp_vertex_bf(P, a, b, d, J, M, g)
    # the vertex enumeration equals the integer DP (no Property 2 assumed) on small values
    for P, a, b, M, g, d, J in _wide_cases(60, 5, 26, 6, 6, rng_h=False):
        d = int(P.sum())
        assert bf.ucddcp_vertex_bf(P, a, b, d, J, M, g) == bf.dp_schedule(P, a, b, d, J, M=M, g=g)
