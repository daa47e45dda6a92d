"""Pins of the oracle's random-number layer, T0 rule, SA (Alg. 1) and DPSO (Alg. 2) loops."""
import math

import numpy as np
import pytest

import gen
import oracle
from tests import bruteforce as bf


# --------------------------------------------------------------------------------- Philox
@pytest.mark.parametrize("ctr,key,expect", [
    # Random123 known-answer vectors for philox4x32_10 (kat_vectors), identical to cuRAND's
    # curand_Philox4x32_10 (curand_philox4x32_x.h); P:220 says the paper drew from cuRand.
    ([0, 0, 0, 0], [0, 0], [0x6627E8D5, 0xE169C58D, 0xBC57AC4C, 0x9B00DBD8]),
    ([0xFFFFFFFF] * 4, [0xFFFFFFFF] * 2, [0x408F276D, 0x41C83B0E, 0xA20BC7C6, 0x6D5451FD]),
    ([0x243F6A88, 0x85A308D3, 0x13198A2E, 0x03707344], [0xA4093822, 0x299F31D0],
     [0xD16CFE09, 0x94FDCCEB, 0x5001E420, 0x24126EA1]),
])
def test_philox_known_answers(ctr, key, expect):
    assert list(oracle.philox4x32_10(ctr, key)) == expect


def test_bnd_and_u01():
    assert oracle.bnd(0, 7) == 0 and oracle.bnd(0xFFFFFFFF, 7) == 6
    assert oracle.bnd(0x80000000, 10) == 5
    assert 0.0 < oracle.u01(0) < 1e-9 and 1 - 1e-9 < oracle.u01(0xFFFFFFFF) < 1.0


# --------------------------------------------------------------------------------- det_exp
def test_det_exp_accuracy_vs_libm():
    xs = np.concatenate([np.linspace(-23.0, 0.0, 200001), -np.logspace(-12, 1.36, 5000)])
    worst = max(abs(oracle.det_exp(x) / math.exp(x) - 1.0) for x in xs)
    assert worst < 1e-15


def test_det_exp_special_points():
    assert oracle.det_exp(0.0) == 1.0
    assert oracle.det_exp(-math.inf) == 0.0
    for k in range(1, 33):  # e^{-k ln2} = 2^-k up to the rounding of the argument k*ln2
        assert abs(oracle.det_exp(-k * math.log(2.0)) * 2.0 ** k - 1.0) < 1e-14


# ------------------------------------------------------------------------ sequences / moves
def test_perm_fy_uniform_n3():
    counts = {}
    N = 12000
    for i in range(N):
        J = tuple(oracle.perm_fy(3, 99, oracle.TAG_SA_INIT, i))
        counts[J] = counts.get(J, 0) + 1
    assert sorted(counts) == sorted(tuple(p) for p in bf.all_sequences(3))
    chi2 = sum((c - N / 6) ** 2 / (N / 6) for c in counts.values())
    assert chi2 < 25.0  # 5 dof, p ~ 1e-4


def test_perm_fy_is_fisher_yates():
    # the first swap uses word 0 of block 0: i = n-1 swaps with bnd(w0, n)
    n, seed, g = 9, 5, 3
    J = oracle.perm_fy(n, seed, oracle.TAG_SA_INIT, g)
    w = oracle.philox4x32_10([0, g, 0, oracle.TAG_SA_INIT << 16], [seed, 0])
    ident = list(range(n))
    j = oracle.bnd(int(w[0]), n)
    ident[n - 1], ident[j] = ident[j], ident[n - 1]
    # replay the remaining swaps with the documented word layout
    q = 1
    for i in range(n - 2, 0, -1):
        ww = oracle.philox4x32_10([q // 4, g, 0, oracle.TAG_SA_INIT << 16], [seed, 0])
        jj = oracle.bnd(int(ww[q % 4]), i + 1)
        ident[i], ident[jj] = ident[jj], ident[i]
        q += 1
    assert list(J) == ident


def test_sa_move_distinct_sorted_uniform():
    n = 6
    subsets, sigmas = {}, {}
    N = 24000
    for k in range(N):
        q, s, u = oracle.sa_move(n, 4, oracle.MOVE_PERT_FY, 17, 2, k)
        assert len(set(q)) == 4 and list(q) == sorted(q) and 0 <= q.min() and q.max() < n
        assert sorted(s) == [0, 1, 2, 3] and 0.0 < u < 1.0
        subsets[tuple(q)] = subsets.get(tuple(q), 0) + 1
        sigmas[tuple(s)] = sigmas.get(tuple(s), 0) + 1
    assert len(subsets) == 15 and len(sigmas) == 24
    e1, e2 = N / 15, N / 24
    assert sum((c - e1) ** 2 / e1 for c in subsets.values()) < 50   # 14 dof
    assert sum((c - e2) ** 2 / e2 for c in sigmas.values()) < 70    # 23 dof


def test_sa_move_small_n_and_swap():
    q, s, _ = oracle.sa_move(3, 4, oracle.MOVE_PERT_FY, 1, 0, 0)
    assert list(q) == [0, 1, 2]
    q, s, _ = oracle.sa_move(1, 4, oracle.MOVE_PERT_FY, 1, 0, 0)
    assert list(q) == [0] and list(s) == [0]
    q, s, _ = oracle.sa_move(10, 4, oracle.MOVE_SWAP, 1, 0, 5)
    assert len(q) == 2 and list(s) == [1, 0]


# ------------------------------------------------------------------------------------- T0
def test_t0_is_population_std():
    inst = gen.cdd_instance(30, 2, 0.4)
    pr = oracle.Problem.from_instance(inst)
    N = 700
    perms = np.stack([oracle.perm_fy(30, 11, oracle.TAG_T0, s) for s in range(N)])
    Z = oracle.eval_batch(pr, perms).astype(np.float64)
    T0 = oracle.t0(pr, oracle.CDD, 11, N)
    assert abs(T0 - np.std(Z)) <= 1e-12 * np.std(Z)


def test_t0_ucddcp_uses_ucddcp_fitness():
    inst = gen.ucddcp_instance(20, 3)
    pr = oracle.Problem.from_instance(inst)
    perms = np.stack([oracle.perm_fy(20, 4, oracle.TAG_T0, s) for s in range(300)])
    Z = oracle.eval_batch(pr, perms, oracle.UCDDCP).astype(np.float64)
    assert abs(oracle.t0(pr, oracle.UCDDCP, 4, 300) - np.std(Z)) <= 1e-12 * np.std(Z)


# ------------------------------------------------------------------------------------- SA
def _sa(n=40, k=1, h=0.4, **kw):
    inst = gen.cdd_instance(n, k, h)
    return inst, oracle.Problem.from_instance(inst), oracle.sa_params(**kw)


def test_sa_zero_steps_returns_initial_sequence():
    inst, pr, p = _sa(steps=0, seed=3)
    r = oracle.sa_chain(pr, p, 100.0, 7)
    J0 = oracle.perm_fy(inst.n, 3, oracle.TAG_SA_INIT, 7)
    assert r["E_best"] == oracle.cdd_eval(pr, J0) and list(r["best"]) == list(J0)


def test_sa_best_is_consistent_and_trace_is_alg1():
    inst, pr, p = _sa(steps=400, seed=5)
    T0 = oracle.t0(pr, oracle.CDD, 5, 500)
    r = oracle.sa_chain(pr, p, T0, 2, trace=True)
    assert oracle.cdd_eval(pr, r["best"]) == r["E_best"]
    assert oracle.cdd_eval(pr, r["final"]) == r["E_final"]
    # replay the trace: E follows accepted E_new; best = min over visited states
    E = oracle.cdd_eval(pr, oracle.perm_fy(inst.n, 5, oracle.TAG_SA_INIT, 2))
    best = E
    for En, acc in zip(r["E_new"], r["accepted"]):
        if En <= E:
            assert acc  # Delta >= 0 always accepted (exp(Delta/T) >= 1 >= rand)
        if acc:
            E = int(En)
            best = min(best, E)
    assert E == r["E_final"] and best == r["E_best"]


def test_sa_zero_temperature_is_greedy():
    inst, pr, p = _sa(steps=300, seed=8)
    r = oracle.sa_chain(pr, p, 0.0, 4, trace=True)
    E = oracle.cdd_eval(pr, oracle.perm_fy(inst.n, 8, oracle.TAG_SA_INIT, 4))
    for En, acc in zip(r["E_new"], r["accepted"]):
        assert bool(acc) == (En <= E)
        if acc:
            E = int(En)


def test_sa_huge_temperature_accepts_everything():
    inst, pr, p = _sa(steps=300, seed=8, mu=1.0)
    r = oracle.sa_chain(pr, p, 1e300, 4, trace=True)
    assert r["accepted"].all()


def test_sa_metropolis_rate_matches_exp():
    # constant T (mu = 1): the acceptance frequency of worsening moves equals E[exp(Delta/T)]
    inst, pr, p = _sa(n=30, steps=6000, seed=21, mu=1.0)
    T = 40.0
    r = oracle.sa_chain(pr, p, T, 0, trace=True)
    E = oracle.cdd_eval(pr, oracle.perm_fy(inst.n, 21, oracle.TAG_SA_INIT, 0))
    probs, accs = [], []
    for En, acc in zip(r["E_new"], r["accepted"]):
        if En > E:
            probs.append(math.exp((E - int(En)) / T))
            accs.append(bool(acc))
        if acc:
            E = int(En)
    probs, accs = np.array(probs), np.array(accs)
    assert len(probs) > 1000
    se = math.sqrt((probs * (1 - probs)).sum()) + 1.0
    assert abs(accs.sum() - probs.sum()) < 5 * se


def test_sa_run_reduces_with_lowest_chain_tie_break():
    inst, pr, p = _sa(n=20, steps=200, seed=2, chains=12, chain_offset=100)
    T0 = oracle.t0(pr, oracle.CDD, 2, 500)
    r = oracle.sa_run(pr, p, T0, chain_best=True)
    cb = r["chain_best"]
    assert r["E_best"] == cb.min() and r["g"] == 100 + int(np.argmin(cb))
    assert oracle.cdd_eval(pr, r["best"]) == r["E_best"]


def test_sa_n10_reaches_the_nfact_optimum():
    # Table II: SA_5000 reaches 0 % deviation at n = 10; here vs the exhaustive optimum
    inst = gen.cdd_instance(10, 1, 0.4)
    pr = oracle.Problem.from_instance(inst)
    z_opt = int(oracle.eval_batch_threaded(pr, gen.all_perms(10)).min())
    p = oracle.sa_params(chains=64, steps=1000, seed=0x5EED0001)
    r = oracle.sa_run(pr, p, oracle.t0(pr, oracle.CDD, 0x5EED0001))
    assert r["E_best"] == z_opt


def test_sa_initial_sequences():
    # initial sequences copied to the device.  Giving each chain its own random sequence
    # explicitly reproduces the default run; zero steps return the given sequence
    inst, pr, p = _sa(n=30, steps=200, seed=6, chains=5, chain_offset=11)
    T0 = oracle.t0(pr, oracle.CDD, 6, 300)
    rows = np.stack([oracle.perm_fy(30, 6, oracle.TAG_SA_INIT, 11 + c) for c in range(5)])
    a = oracle.sa_run(pr, p, T0, chain_best=True)
    b = oracle.sa_run(pr, oracle.sa_params(chains=5, steps=200, seed=6, chain_offset=11, init=rows),
                      T0, chain_best=True)
    assert np.array_equal(a["chain_best"], b["chain_best"]) and np.array_equal(a["best"], b["best"])
    v = np.argsort(inst.P / inst.alpha).astype(np.int16)
    z = oracle.cdd_eval(pr, v)
    r = oracle.sa_chain(pr, oracle.sa_params(chains=1, steps=0, seed=6, init=v), T0, 0)
    assert r["E_best"] == z and np.array_equal(r["best"], v)
    r = oracle.sa_chain(pr, oracle.sa_params(chains=1, steps=300, seed=6, init=v), T0, 0)
    assert r["E_best"] <= z


# ---------------------------------------------------------------------- synchronous SA (F2)
def test_sa_sync_single_chain_unit_length_is_the_async_chain():
    # chains = 1, M = 1: level j is one move at T0*mu^j from the previous final state with the
    # counters of step j -- exactly Alg. 1 (cooling every step)
    inst, pr, p = _sa(n=40, steps=1, seed=5)
    T0 = oracle.t0(pr, oracle.CDD, 5, 400)
    L = 700
    s = oracle.sa_sync(pr, p, T0, L)
    pa = oracle.sa_params(chains=1, steps=L, seed=5)
    a = oracle.sa_chain(pr, pa, T0, 0, trace=True)
    assert s["E_best"] == a["E_best"] and s["g"] == 0
    assert oracle.cdd_eval(pr, s["best"]) == s["E_best"]
    # the level minimum is the chain's state after each step
    E, states = oracle.cdd_eval(pr, oracle.perm_fy(inst.n, 5, oracle.TAG_SA_INIT, 0)), []
    for En, acc in zip(a["E_new"], a["accepted"]):
        E = int(En) if acc else E
        states.append(E)
    assert np.array_equal(s["level_min_E"], np.array(states))


def test_sa_sync_one_level_is_async_at_constant_temperature():
    inst, pr, p = _sa(n=30, steps=250, seed=9, chains=10, chain_offset=7)
    r = oracle.sa_sync(pr, p, 60.0, 1)
    pa = oracle.sa_params(chains=10, steps=250, seed=9, chain_offset=7, mu=1.0)
    a = oracle.sa_run(pr, pa, 60.0)
    assert (r["E_best"], r["g"]) == (a["E_best"], a["g"]) and np.array_equal(r["best"], a["best"])
    finals = [oracle.sa_chain(pr, pa, 60.0, 7 + c)["E_final"] for c in range(10)]
    assert r["level_min_E"][0] == min(finals) and r["level_min_g"][0] == 7 + int(np.argmin(finals))


def test_sa_sync_greedy_levels_never_worsen_and_n10_optimum():
    inst, pr, p = _sa(n=25, steps=40, seed=3, chains=8)
    r = oracle.sa_sync(pr, p, 0.0, 30)  # T = 0: only non-worsening moves
    assert np.all(np.diff(r["level_min_E"]) <= 0)
    assert r["E_best"] == r["level_min_E"].min() == oracle.cdd_eval(pr, r["best"])
    inst = gen.cdd_instance(10, 1, 0.4)
    pr = oracle.Problem.from_instance(inst)
    z_opt = int(oracle.eval_batch_threaded(pr, gen.all_perms(10)).min())
    p = oracle.sa_params(chains=32, steps=20, seed=0x5EED0002)
    r = oracle.sa_sync(pr, p, oracle.t0(pr, oracle.CDD, 0x5EED0002), 60)
    assert r["E_best"] == z_opt


# ----------------------------------------------------------------------------------- DPSO
def test_dpso_operators():
    rng = np.random.default_rng(3)
    for t in range(300):
        n = int(rng.integers(2, 30))
        p = rng.permutation(n).astype(np.int16)
        pb = rng.permutation(n).astype(np.int16)
        g = rng.permutation(n).astype(np.int16)
        w = [int(x) for x in rng.integers(0, 2**32, 3, dtype=np.uint64)]
        f1 = oracle.dpso_f1(p, w[0], w[1])
        diff = np.nonzero(f1 != p)[0]
        assert sorted(f1) == list(range(n)) and len(diff) == 2
        assert f1[diff[0]] == p[diff[1]] and f1[diff[1]] == p[diff[0]]
        f2 = oracle.dpso_f2(p, pb, w[2])
        c = 1 + oracle.bnd(w[2], n - 1)
        assert list(f2[:c]) == list(p[:c])
        assert list(f2[c:]) == [j for j in pb if j not in set(p[:c].tolist())]
        f3 = oracle.dpso_f3(p, g, w[0], w[1])
        a = oracle.bnd(w[0], n - 1)
        b = oracle.bnd(w[1], n)
        b = n - 1 if b == a else b
        q0, q1 = min(a, b), max(a, b)
        assert list(f3[q0:q1 + 1]) == list(p[q0:q1 + 1])
        kept = set(p[q0:q1 + 1].tolist())
        rest = [j for j in g if j not in kept]
        assert list(f3[:q0]) + list(f3[q1 + 1:]) == rest


def test_dpso_without_operators_returns_best_initial():
    inst = gen.cdd_instance(25, 2, 0.6)
    pr = oracle.Problem.from_instance(inst)
    p = oracle.dpso_params(particles=40, iters=30, w=0.0, c1=0.0, c2=0.0, seed=9)
    r = oracle.dpso_run(pr, p, trace=True)
    Z0 = [oracle.cdd_eval(pr, oracle.perm_fy(25, 9, oracle.TAG_DPSO_INIT, i)) for i in range(40)]
    assert r["E_best"] == min(Z0) and r["id"] == int(np.argmin(Z0))
    assert (r["gbest_trace"] == min(Z0)).all()


def test_dpso_gbest_monotone_and_valid():
    inst = gen.cdd_instance(30, 4, 0.4)
    pr = oracle.Problem.from_instance(inst)
    p = oracle.dpso_params(particles=32, iters=60, seed=12)
    r = oracle.dpso_run(pr, p, trace=True)
    tr = r["gbest_trace"]
    assert (np.diff(tr) <= 0).all() and r["E_best"] <= tr[-1]
    assert sorted(r["best"]) == list(range(30))
    assert oracle.cdd_eval(pr, r["best"]) == r["E_best"]


def test_dpso_n10_reaches_optimum():
    inst = gen.cdd_instance(10, 1, 0.4)
    pr = oracle.Problem.from_instance(inst)
    z_opt = int(oracle.eval_batch_threaded(pr, gen.all_perms(10)).min())
    r = oracle.dpso_run(pr, oracle.dpso_params(particles=128, iters=200, seed=5))
    assert r["E_best"] == z_opt


# ------------------------------------------------------------ insertion and window moves
def test_insert_move_is_uniform_ordered_pair():
    # BASELINE north_star "swap/insertion move" (R11b): (from, to) are two distinct positions in
    # the order of the two Floyd draws -- every ordered pair of distinct positions equally likely
    n, N = 5, 40000
    counts = {}
    for k in range(N):
        q, s, u = oracle.sa_move(n, 4, oracle.MOVE_INSERT, 23, 1, k)
        assert len(q) == 2 and q[0] != q[1] and 0 <= q.min() and q.max() < n and 0.0 < u < 1.0
        counts[tuple(q)] = counts.get(tuple(q), 0) + 1
    assert len(counts) == n * (n - 1)
    e = N / (n * (n - 1))
    assert sum((c - e) ** 2 / e for c in counts.values()) < 60  # 19 dof


def test_insert_neighbour_definition():
    # insertion: the moved job lands at `to`, and deleting it from both sequences leaves the same
    # sequence (every other job keeps its relative order) -- checked against that definition
    rng = np.random.default_rng(7)
    for t in range(400):
        n = int(rng.integers(2, 40))
        s = rng.permutation(n).astype(np.int16)
        k = int(rng.integers(0, 1 << 30))
        q, sig, _ = oracle.sa_move(n, 4, oracle.MOVE_INSERT, 3, 9, k)
        f, to = int(q[0]), int(q[1])
        s2 = oracle.sa_neighbour(s, oracle.MOVE_INSERT, q, sig)
        assert sorted(s2.tolist()) == list(range(n))
        assert s2[to] == s[f]
        assert [x for x in s2.tolist() if x != s[f]] == [x for x in s.tolist() if x != s[f]]
        lo, hi = min(f, to), max(f, to)
        assert np.array_equal(s2[:lo], s[:lo]) and np.array_equal(s2[hi + 1:], s[hi + 1:])


def test_window_move_contiguous_uniform():
    # "A sub-sequence of size Pert=4 is selected ... Fisher Yates ... on this sub-sequence
    # while retaining the position of other jobs" (R11c)
    n, N = 9, 30000
    starts, sigmas = {}, {}
    rng = np.random.default_rng(1)
    for k in range(N):
        q, sig, u = oracle.sa_move(n, 4, oracle.MOVE_WINDOW, 31, 4, k)
        assert list(q) == list(range(q[0], q[0] + 4)) and q[-1] < n
        assert sorted(sig) == [0, 1, 2, 3]
        starts[int(q[0])] = starts.get(int(q[0]), 0) + 1
        sigmas[tuple(sig)] = sigmas.get(tuple(sig), 0) + 1
        if k < 300:
            s = rng.permutation(n).astype(np.int16)
            s2 = oracle.sa_neighbour(s, oracle.MOVE_WINDOW, q, sig)
            out = np.ones(n, bool)
            out[q] = False
            assert np.array_equal(s2[out], s[out]) and sorted(s2[q]) == sorted(s[q])
    assert len(starts) == n - 3 and len(sigmas) == 24
    e1, e2 = N / (n - 3), N / 24
    assert sum((c - e1) ** 2 / e1 for c in starts.values()) < 30   # 5 dof
    assert sum((c - e2) ** 2 / e2 for c in sigmas.values()) < 70   # 23 dof
    # Pert-FY and window share the slot shuffle words (same sigma for the same step)
    for k in range(50):
        assert list(oracle.sa_move(n, 4, oracle.MOVE_WINDOW, 31, 4, k)[1]) == \
            list(oracle.sa_move(n, 4, oracle.MOVE_PERT_FY, 31, 4, k)[1])


@pytest.mark.parametrize("move", [oracle.MOVE_INSERT, oracle.MOVE_WINDOW])
def test_sa_chain_with_other_moves_is_alg1(move):
    inst, pr, p = _sa(n=35, steps=500, seed=13, move=move)
    T0 = oracle.t0(pr, oracle.CDD, 13, 400)
    r = oracle.sa_chain(pr, p, T0, 3, trace=True)
    assert oracle.cdd_eval(pr, r["best"]) == r["E_best"]
    # replay with the oracle's own move + neighbour: every E_new is the penalty of the neighbour
    s = oracle.perm_fy(inst.n, 13, oracle.TAG_SA_INIT, 3)
    for k, (En, acc) in enumerate(zip(r["E_new"], r["accepted"])):
        q, sig, _ = oracle.sa_move(inst.n, 4, move, 13, 3, k)
        s_new = oracle.sa_neighbour(s, move, q, sig)
        assert oracle.cdd_eval(pr, s_new) == En
        if acc:
            s = s_new
    assert np.array_equal(s, r["final"])


@pytest.mark.parametrize("move", [oracle.MOVE_INSERT, oracle.MOVE_WINDOW])
def test_sa_other_moves_reach_n10_optimum(move):
    inst = gen.cdd_instance(10, 1, 0.4)
    pr = oracle.Problem.from_instance(inst)
    z_opt = int(oracle.eval_batch_threaded(pr, gen.all_perms(10)).min())
    p = oracle.sa_params(chains=64, steps=1000, seed=0x5EED0001, move=move)
    r = oracle.sa_run(pr, p, oracle.t0(pr, oracle.CDD, 0x5EED0001))
    assert r["E_best"] == z_opt
