"""GPU parity: T0 rule and SA chains replayed step by step against the oracle (bit-exact)."""
import os

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


def _prob(inst):
    return oracle.Problem.from_instance(inst)


@pytest.mark.parametrize("n,problem", [(5, "cdd"), (10, "cdd"), (33, "cdd"), (100, "cdd"),
                                       (200, "ucddcp"), (500, "cdd"), (1000, "cdd"),
                                       (1000, "ucddcp")])
def test_t0_bit_exact(lib, n, problem):
    inst = gen.ucddcp_instance(n, 3) if problem == "ucddcp" else gen.cdd_instance(n, 3, 0.4)
    ins = lib.Instance.from_gen(inst)
    samples = 5000 if n <= 200 else 1500
    t_gpu = float(lib.sa_t0(ins, problem, seed=123, samples=samples).item())
    t_ref = oracle.t0(_prob(inst), oracle.CDD if problem == "cdd" else oracle.UCDDCP, 123, samples)
    assert t_gpu == t_ref  # same double, bit for bit


ORACLE_MOVES = {"pert_fy": oracle.MOVE_PERT_FY, "swap": oracle.MOVE_SWAP,
                "insert": oracle.MOVE_INSERT, "window": oracle.MOVE_WINDOW}

# threads per chain: 32 = warp kernel, 16 / 8 / 4 = group kernel (2 / 4 / 8 chains per warp)
LANES = [32, 16, 8, 4]


def _lanes_ok(n, lanes):
    return lanes != 4 or n <= 256


def _run_both(lib, inst, problem, chains, steps, seed, T0=0.0, samples=5000, move="pert_fy",
              pert=4, chain_offset=0, trace=True, mu=0.88, lanes=0):
    import torch

    ins = lib.Instance.from_gen(inst)
    res = lib.sa_run(ins, chains, steps, problem=problem, mu=mu, T0=T0, t0_samples=samples,
                     pert=pert, move=move, seed=seed, chain_offset=chain_offset, trace=trace,
                     chain_best=True, chain_final=True, lanes=lanes)
    torch.cuda.synchronize()
    pen, perm, gid = lib.best_get(ins)
    pr = _prob(inst)
    P = oracle.CDD if problem == "cdd" else oracle.UCDDCP
    T0_ref = T0 if T0 > 0 else oracle.t0(pr, P, seed, samples)
    assert float(res["T0"].item()) == T0_ref
    p = oracle.sa_params(problem=P, chains=chains, steps=steps, mu=mu, pert=pert,
                         move=ORACLE_MOVES[move], seed=seed, chain_offset=chain_offset)
    return ins, res, (pen, perm, gid), pr, p, T0_ref


def test_config1_single_chain_10k_steps_trace(lib):
    # BASELINE config 1: one 10k-step SA chain at n=10 (T underflows to 0 at ~5900 steps)
    inst = gen.cdd_instance(10, 1, 0.4)
    seed = 0x5EED0001
    ins, res, (pen, perm, gid), pr, p, T0 = _run_both(lib, inst, "cdd", 1, 10000, seed)
    ref = oracle.sa_chain(pr, p, T0, 0, trace=True)
    tr = res["trace"].cpu().numpy()[0]
    assert np.array_equal(tr >> 1, ref["E_new"])
    assert np.array_equal((tr & 1).astype(bool), ref["accepted"])
    assert pen == ref["E_best"] and gid == 0 and np.array_equal(perm, ref["best"])
    assert int(res["chain_final"].item()) == ref["E_final"]


@pytest.mark.parametrize("lanes", LANES)
@pytest.mark.parametrize("n,chains,steps", [(4, 40, 300), (17, 64, 400), (100, 256, 2000),
                                            (250, 96, 500), (600, 40, 300), (1000, 32, 300)])
def test_many_chains_trace_parity(lib, n, chains, steps, lanes):
    if not _lanes_ok(n, lanes):
        pytest.skip("lanes=4 needs n <= 256")
    inst = gen.cdd_instance(n, 2, 0.6)
    seed = 1000 + n
    ins, res, (pen, perm, gid), pr, p, T0 = _run_both(lib, inst, "cdd", chains, steps, seed,
                                                     samples=800, lanes=lanes)
    tr = res["trace"].cpu().numpy()
    cb = res["chain_best"].cpu().numpy()
    cf = res["chain_final"].cpu().numpy()
    for c in range(chains):
        ref = oracle.sa_chain(pr, p, T0, c, trace=True)
        assert np.array_equal(tr[c] >> 1, ref["E_new"]), c
        assert np.array_equal((tr[c] & 1).astype(bool), ref["accepted"]), c
        assert cb[c] == ref["E_best"] and cf[c] == ref["E_final"], c
    full = oracle.sa_run(pr, p, T0)
    assert (pen, gid) == (full["E_best"], full["g"])
    assert np.array_equal(perm, full["best"])


@pytest.mark.parametrize("lanes", LANES)
@pytest.mark.parametrize("n,chains,steps", [(40, 32, 300), (200, 48, 400), (333, 40, 200),
                                            (1000, 20, 150)])
def test_ucddcp_sa_parity(lib, n, chains, steps, lanes):
    if not _lanes_ok(n, lanes):
        pytest.skip("lanes=4 needs n <= 256")
    inst = gen.ucddcp_instance(n, 4)
    ins, res, (pen, perm, gid), pr, p, T0 = _run_both(lib, inst, "ucddcp", chains, steps, 77,
                                                     samples=600, lanes=lanes)
    cb = res["chain_best"].cpu().numpy()
    tr = res["trace"].cpu().numpy()
    for c in range(chains):
        ref = oracle.sa_chain(pr, p, T0, c, trace=True)
        assert np.array_equal(tr[c] >> 1, ref["E_new"]) and cb[c] == ref["E_best"], c
    full = oracle.sa_run(pr, p, T0)
    assert (pen, gid) == (full["E_best"], full["g"]) and np.array_equal(perm, full["best"])
    assert oracle.ucddcp_eval(pr, perm) == pen


@pytest.mark.parametrize("lanes", [32, 8, 4])
@pytest.mark.parametrize("move,pert", [("swap", 4), ("pert_fy", 2), ("pert_fy", 3), ("pert_fy", 1)])
def test_move_variants(lib, move, pert, lanes):
    inst = gen.cdd_instance(60, 5, 0.2)
    ins, res, (pen, perm, gid), pr, p, T0 = _run_both(lib, inst, "cdd", 32, 300, 5, move=move,
                                                     pert=pert, samples=300, lanes=lanes)
    tr = res["trace"].cpu().numpy()
    for c in range(32):
        ref = oracle.sa_chain(pr, p, T0, c, trace=True)
        assert np.array_equal(tr[c] >> 1, ref["E_new"]), c
    full = oracle.sa_run(pr, p, T0)
    assert (pen, gid) == (full["E_best"], full["g"])


@pytest.mark.parametrize("lanes", LANES)
@pytest.mark.parametrize("move", ["insert", "window"])
@pytest.mark.parametrize("n,problem,chains,steps,mu", [
    (2, "cdd", 16, 50, 0.88), (9, "cdd", 24, 300, 1.0), (64, "cdd", 40, 400, 1.0),
    (130, "ucddcp", 24, 300, 1.0), (257, "cdd", 24, 300, 0.995), (1000, "cdd", 12, 200, 1.0),
    (700, "ucddcp", 12, 150, 1.0)])
def test_insert_and_window_moves(lib, move, n, problem, chains, steps, mu, lanes):
    # insertion (R11b) and contiguous-window (R11c) moves: every chain's trace, best and
    # final penalty replayed by the oracle; constant temperature keeps many uphill acceptances
    # (id rotations, best-state copies) in the run
    if not _lanes_ok(n, lanes):
        pytest.skip("lanes=4 needs n <= 256")
    inst = gen.ucddcp_instance(n, 6) if problem == "ucddcp" else gen.cdd_instance(n, 6, 0.4)
    ins, res, (pen, perm, gid), pr, p, T0 = _run_both(lib, inst, problem, chains, steps, 31 + n,
                                                     move=move, samples=300, mu=mu, lanes=lanes)
    tr = res["trace"].cpu().numpy()
    cb = res["chain_best"].cpu().numpy()
    cf = res["chain_final"].cpu().numpy()
    for c in range(chains):
        ref = oracle.sa_chain(pr, p, T0, c, trace=True)
        assert np.array_equal(tr[c] >> 1, ref["E_new"]), c
        assert np.array_equal((tr[c] & 1).astype(bool), ref["accepted"]), c
        assert cb[c] == ref["E_best"] and cf[c] == ref["E_final"], c
    full = oracle.sa_run(pr, p, T0)
    assert (pen, gid) == (full["E_best"], full["g"]) and np.array_equal(perm, full["best"])


@pytest.mark.parametrize("move", ["insert", "window"])
def test_other_moves_no_trace_full_grid(lib, move):
    # the non-trace kernels (bench configuration) with enough chains for the automatic layout
    import torch

    inst = gen.cdd_instance(300, 2, 0.6)
    ins = lib.Instance.from_gen(inst)
    chains, steps = 4096, 60
    res = lib.sa_run(ins, chains, steps, move=move, seed=77, T0=500.0, chain_best=True,
                     chain_final=True)
    torch.cuda.synchronize()
    pen, perm, gid = lib.best_get(ins)
    pr = _prob(inst)
    p = oracle.sa_params(chains=chains, steps=steps, move=ORACLE_MOVES[move], seed=77)
    cb = res["chain_best"].cpu().numpy()
    cf = res["chain_final"].cpu().numpy()
    for c in list(range(0, chains, 97)) + [chains - 1]:
        ref = oracle.sa_chain(pr, p, 500.0, c)
        assert cb[c] == ref["E_best"] and cf[c] == ref["E_final"], c
    assert oracle.cdd_eval(pr, perm) == pen == cb.min() and gid == int(np.argmin(cb))


def test_explicit_T0_and_constant_temperature(lib):
    inst = gen.cdd_instance(80, 6, 0.4)
    ins, res, (pen, perm, gid), pr, p, T0 = _run_both(lib, inst, "cdd", 16, 1500, 9, T0=350.0,
                                                     mu=1.0)
    tr = res["trace"].cpu().numpy()
    acc_worse = 0
    for c in range(16):
        ref = oracle.sa_chain(pr, p, T0, c, trace=True)
        assert np.array_equal(tr[c] >> 1, ref["E_new"]) and np.array_equal(
            (tr[c] & 1).astype(bool), ref["accepted"]), c
        acc_worse += int(ref["accepted"].sum())
    assert acc_worse > 0


def test_sharding_invariance(lib):
    # T10: the global best over R emulated ranks (chain_offset = r*C) equals one run of R*C chains
    inst = gen.cdd_instance(100, 7, 0.4)
    R, Cc, steps, seed = 4, 64, 200, 31
    ins = lib.Instance.from_gen(inst)
    best = []
    for r in range(R):
        lib.sa_run(ins, Cc, steps, seed=seed, chain_offset=r * Cc, t0_samples=500)
        pen, perm, gid = lib.best_get(ins)
        best.append((pen, gid, perm.copy()))
    lib.sa_run(ins, R * Cc, steps, seed=seed, t0_samples=500)
    pen, perm, gid = lib.best_get(ins)
    m = min(best, key=lambda t: (t[0], t[1]))
    assert (m[0], m[1]) == (pen, gid) and np.array_equal(m[2], perm)


def test_large_chain_count_best_matches_oracle_chain(lib):
    # many more chains than resident warps (persistent loop); best re-verified by the oracle
    import torch

    inst = gen.cdd_instance(1000, 1, 0.4)
    ins = lib.Instance.from_gen(inst)
    res = lib.sa_run(ins, 20000, 60, seed=5, chain_best=True, t0_samples=600)
    torch.cuda.synchronize()
    pen, perm, gid = lib.best_get(ins)
    pr = _prob(inst)
    assert oracle.cdd_eval(pr, perm) == pen
    cb = res["chain_best"].cpu().numpy()
    assert pen == cb.min() and gid == int(np.argmin(cb))
    T0 = float(res["T0"].item())
    p = oracle.sa_params(chains=1, steps=60, seed=5)
    for c in [0, 1, 4095, 4096, 12345, 19999, gid]:
        assert oracle.sa_chain(pr, p, T0, c)["E_best"] == cb[c], c


# Edge cases (within the ABI's packed-record limits, cdd.h) of the group kernel's boundary search (one case per rows-per-lane size E = 8..64):
# sum p > 2^16 (row-relative packing), zero penalties (every alpha 0: k0 = n; every beta 0),
# Btot near the 2^16 limit of the ABI, d = 0 and d >= sum p.
EDGE = [
    (70, dict(p=(1, 255), alpha=(0, 15), beta=(0, 15), h=0.5)),
    (150, dict(p=(1, 4), alpha=(0, 0), beta=(1, 9), h=0.3)),
    (150, dict(p=(1, 9), alpha=(1, 9), beta=(0, 0), h=0.6)),
    (400, dict(p=(1, 4), alpha=(100, 127), beta=(100, 127), h=0.4)),
    (700, dict(p=(1, 255), alpha=(0, 15), beta=(0, 15), h=0.2)),
    (700, dict(p=(1, 20), alpha=(1, 10), beta=(1, 15), h=0.0)),
    (1000, dict(p=(1, 20), alpha=(1, 10), beta=(1, 15), h=1.2)),
    (1000, dict(p=(1, 3), alpha=(40, 60), beta=(40, 60), h=0.45)),
    # alpha + beta in [78, 85]: the quad form of the boundary row's level 1 at its byte limit
    # (three prefix bytes of 85 = 255); the case above (alpha + beta up to 120) takes the pairs
    (1000, dict(p=(1, 3), alpha=(40, 45), beta=(38, 40), h=0.5)),
    (600, dict(p=(1, 3), alpha=(40, 45), beta=(38, 40), h=0.9)),
]


@pytest.mark.parametrize("lanes", [0] + LANES)
@pytest.mark.parametrize("n,kw", EDGE)
@pytest.mark.parametrize("problem", ["cdd", "ucddcp"])
def test_edge_instances_trace_parity(lib, n, kw, problem, lanes):
    if problem == "ucddcp" and kw["alpha"][1] == 0:
        pytest.skip("UCDDCP gamma range needs alpha > 0")
    if not _lanes_ok(n, lanes):
        pytest.skip("lanes=4 needs n <= 256")
    inst = gen.ranged_instance(n, 9, problem=problem, **kw)
    chains = 24
    if problem == "ucddcp" and lib.Instance.from_gen(inst).query()["ucddcp_generic"] and lanes in (4, 8, 16):
        # M, P-M, gamma do not fit the packed UCDDCP record: the UCDDCP runs on the generic path
        # (one warp per chain), the group layouts refuse it
        with pytest.raises(lib.CddError):
            lib.sa_run(lib.Instance.from_gen(inst), 4, 10, problem="ucddcp", T0=1.0, lanes=lanes)
        return
    ins, res, (pen, perm, gid), pr, p, T0 = _run_both(lib, inst, problem, chains, 120, 31 + n,
                                                     samples=200, lanes=lanes)
    tr = res["trace"].cpu().numpy()
    for c in range(chains):
        ref = oracle.sa_chain(pr, p, T0, c, trace=True)
        assert np.array_equal(tr[c] >> 1, ref["E_new"]), c
        assert np.array_equal((tr[c] & 1).astype(bool), ref["accepted"]), c
    full = oracle.sa_run(pr, p, T0)
    assert (pen, gid) == (full["E_best"], full["g"]) and np.array_equal(perm, full["best"])


def test_lanes_argument_checks(lib):
    big = gen.cdd_instance(300, 1, 0.4)
    with pytest.raises(lib.CddError):
        lib.sa_run(lib.Instance.from_gen(big), 64, 10, T0=5.0, lanes=4)  # n > 256
    with pytest.raises(lib.CddError):
        lib.sa_run(lib.Instance.from_gen(big), 64, 10, T0=5.0, lanes=12)
    # alpha > 255: no 16-bit records, the group layouts refuse, the warp layout runs
    heavy = gen.ranged_instance(80, 3, p=(1, 3), alpha=(200, 400), beta=(1, 5), h=0.5)
    ins = lib.Instance.from_gen(heavy)
    with pytest.raises(lib.CddError):
        lib.sa_run(ins, 64, 10, T0=5.0, lanes=8)
    lib.sa_run(ins, 64, 10, T0=5.0, lanes=32)
    lib.sa_run(ins, 4096, 10, T0=5.0)  # automatic: warp layout
    pen, perm, gid = lib.best_get(ins)
    assert oracle.cdd_eval(_prob(heavy), perm) == pen


def test_sa_layout_query(lib):
    for n, chains, lanes in [(1000, 65536, 0), (100, 16384, 0), (100, 100, 0), (300, 4096, 16),
                             (50, 8192, 4), (700, 2048, 32)]:
        ins = lib.Instance.from_gen(gen.cdd_instance(n, 1, 0.4))
        g, e = lib.sa_layout(ins, chains, lanes=lanes)
        assert g in (4, 8, 16, 32) and g * e >= n and (lanes == 0 or g == lanes)
        if chains < 1024:
            assert g == 32
    # automatic choices measured fastest (profiles/r1_fig11_sweep_cdd_n1000.txt,
    # profiles/r1b_fig11_sweep_cdd_n100.txt)
    for n, chains, want in [(1000, 65536, 8), (1000, 4096, 16), (100, 65536, 4), (100, 16384, 4),
                            (100, 4096, 8)]:
        ins = lib.Instance.from_gen(gen.cdd_instance(n, 1, 0.4))
        assert lib.sa_layout(ins, chains)[0] == want, (n, chains)


def test_bench_config_sampled_parity(lib):
    # the BASELINE headline configuration exactly as bench.py launches it (config 5, h = 0.4:
    # n = 1000, 65536 chains x 5000 steps, T0 from 5000 samples, automatic layout); the oracle
    # replays sampled chains one by one, the global best is re-evaluated
    import torch

    import bench

    inst = gen.cdd_instance(bench.N_JOBS, bench.INSTANCE_SEED, 0.4)
    ins = lib.Instance.from_gen(inst)
    T0 = lib.sa_t0(ins, "cdd", seed=bench.RUN_SEED, samples=bench.T0_SAMPLES)
    res = lib.sa_run(ins, bench.CHAINS, bench.SA_STEPS, seed=bench.RUN_SEED, T0_dev=T0,
                     chain_best=True, chain_final=True)
    torch.cuda.synchronize()
    pen, perm, gid = lib.best_get(ins)
    cb = res["chain_best"].cpu().numpy()
    cf = res["chain_final"].cpu().numpy()
    pr = _prob(inst)
    assert oracle.cdd_eval(pr, perm) == pen == cb.min() and gid == int(np.argmin(cb))
    T0v = float(T0.item())
    assert T0v == oracle.t0(pr, oracle.CDD, bench.RUN_SEED, bench.T0_SAMPLES)
    p = oracle.sa_params(chains=1, steps=bench.SA_STEPS, seed=bench.RUN_SEED)
    # 1024 sampled chains (edges of warps, CTAs and rounds, the winner, the rest seeded-random),
    # replayed by the oracle on the host threads (ctypes releases the GIL)
    rng = np.random.default_rng(5)
    sample = sorted(set([0, 1, 3, 4, 31, 32, 4096, 40000, bench.CHAINS - 1, gid] +
                        rng.choice(bench.CHAINS, 1014, replace=False).tolist()))
    got = {}

    def work(cs):
        for c in cs:
            r = oracle.sa_chain(pr, p, T0v, c)
            got[c] = (r["E_best"], r["E_final"])

    import threading

    nt = max(1, min(16, os.cpu_count() or 1))
    ts = [threading.Thread(target=work, args=(sample[i::nt],)) for i in range(nt)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    for c in sample:
        assert got[c] == (cb[c], cf[c]), c


def test_configs_2_3_sampled_parity(lib):
    # BASELINE configs 2 and 3 exactly as bench.py launches them (automatic layouts, T0 from 5000
    # samples inside sa_run): config 2 = CDD n=100, instance 1, every h, 4096 chains x 5000 steps
    # plus the 2^20-sequence batched evaluation; config 3 = UCDDCP n=200 (d = sum p), 16384 chains
    # x 5000 steps.  The oracle recomputes T0, replays sampled chains and evaluates sampled rows.
    import torch

    p2 = gen.random_perms_device(1 << 20, 100, 2)
    rows = [0, 1, 777, 123456, 524287, (1 << 20) - 1]
    sample = p2[rows].cpu().numpy()
    for h in gen.H_VALUES:
        inst = gen.cdd_instance(100, 1, h)
        ins = lib.Instance.from_gen(inst)
        pr = _prob(inst)
        z = lib.cdd_eval_batch(ins, p2).cpu().numpy()
        assert np.array_equal(z[rows], oracle.eval_batch(pr, sample)), h
        res = lib.sa_run(ins, 4096, 5000, seed=0x5EED0002, chain_best=True)
        torch.cuda.synchronize()
        T0 = float(res["T0"].item())
        assert T0 == oracle.t0(pr, oracle.CDD, 0x5EED0002, 5000), h
        cb = res["chain_best"].cpu().numpy()
        pen, perm, gid = lib.best_get(ins)
        assert pen == cb.min() and gid == int(np.argmin(cb)) and oracle.cdd_eval(pr, perm) == pen
        p = oracle.sa_params(chains=1, steps=5000, seed=0x5EED0002)
        for c in [0, 2049, 4095, gid]:
            assert oracle.sa_chain(pr, p, T0, c)["E_best"] == cb[c], (h, c)
    inst = gen.ucddcp_instance(200, 1)
    ins = lib.Instance.from_gen(inst)
    pr = _prob(inst)
    res = lib.sa_run(ins, 16384, 5000, problem="ucddcp", seed=0x5EED0003, chain_best=True)
    torch.cuda.synchronize()
    T0 = float(res["T0"].item())
    assert T0 == oracle.t0(pr, oracle.UCDDCP, 0x5EED0003, 5000)
    cb = res["chain_best"].cpu().numpy()
    pen, perm, gid = lib.best_get(ins)
    assert pen == cb.min() and gid == int(np.argmin(cb))
    p = oracle.sa_params(problem=oracle.UCDDCP, chains=1, steps=5000, seed=0x5EED0003)
    for c in [0, 8191, 16383, gid]:
        assert oracle.sa_chain(pr, p, T0, c)["E_best"] == cb[c], c


@pytest.mark.parametrize("problem,n,chains,steps", [("cdd", 200, 16000, 200), ("ucddcp", 200, 16384, 150),
                                                    ("cdd", 120, 15000, 37)])
def test_balanced_schedule_every_chain(lib, problem, n, chains, steps):
    # more chains than resident slots but a mostly empty last round: the balanced schedule splits
    # chains between two warps (state handed over mid-run); every chain's best and final penalty,
    # the winner and its sequence must equal the oracle's replay -- and the round-robin run
    import os
    import torch

    inst = gen.ucddcp_instance(n, 2) if problem == "ucddcp" else gen.cdd_instance(n, 2, 0.4)
    ins = lib.Instance.from_gen(inst)
    res = lib.sa_run(ins, chains, steps, problem=problem, seed=77, T0=2500.0, lanes=8,
                     chain_best=True, chain_final=True)
    torch.cuda.synchronize()
    cb, cf = res["chain_best"].cpu().numpy(), res["chain_final"].cpu().numpy()
    pen, perm, gid = lib.best_get(ins)
    pr = _prob(inst)
    code = oracle.UCDDCP if problem == "ucddcp" else oracle.CDD
    p = oracle.sa_params(problem=code, chains=1, steps=steps, seed=77)
    for c in range(chains):
        r = oracle.sa_chain(pr, p, 2500.0, c)
        assert (r["E_best"], r["E_final"]) == (cb[c], cf[c]), c
    assert pen == cb.min() and gid == int(np.argmin(cb))
    assert np.array_equal(perm, oracle.sa_chain(pr, p, 2500.0, gid)["best"])
    os.environ["CDD_SA_BALANCE"] = "0"
    try:
        r2 = lib.sa_run(ins, chains, steps, problem=problem, seed=77, T0=2500.0, lanes=8, chain_best=True)
        torch.cuda.synchronize()
        assert np.array_equal(r2["chain_best"].cpu().numpy(), cb)
    finally:
        del os.environ["CDD_SA_BALANCE"]


# The nibble layout with sub-block summaries (csrc/sa_nib.cuh): CDD with alpha, beta <= 15 and
# pmax * max(alpha, beta) * 120 < 2^16 at G = 8, E = 128 (n in (512, 1024]; 16-position sub-blocks)
# or E = 64 (n in (256, 512]; 8-position sub-blocks).  Every move of <= 4
# positions (insertion keeps the byte rows at this layout: the same check covers it), traced chain
# by chain against the oracle, and the same run with the byte-row layout
# (CDD_SA_NO_NIB=1) must give the identical trace.  The instances put the 16-bit sub-block forms
# at their limit (p up to 36 with weights 15: 36 * 15 * 120 = 64800) and n off the sub-block grid.
NIB = [
    (1000, dict(p=(1, 20), alpha=(1, 10), beta=(1, 15), h=0.4)),
    (777, dict(p=(30, 36), alpha=(14, 15), beta=(13, 15), h=0.6)),
    (530, dict(p=(1, 36), alpha=(0, 15), beta=(0, 15), h=0.2)),
    # edges: n just above E = 64 (lanes 5-7 hold padding), n = 1024 (no padding), zero weights,
    # d = 0 and d >= sum p, every value at the layout's limit (acc = 36 * 15 * 120 = 64800)
    (513, dict(p=(1, 20), alpha=(0, 0), beta=(1, 15), h=0.0)),
    (1024, dict(p=(1, 20), alpha=(1, 15), beta=(0, 0), h=1.2)),
    (1024, dict(p=(36, 36), alpha=(15, 15), beta=(15, 15), h=0.5)),
    # 8-position sub-blocks at E = 64 (n in (256, 512])
    (500, dict(p=(1, 20), alpha=(1, 10), beta=(1, 15), h=0.6)),
    (257, dict(p=(30, 36), alpha=(0, 15), beta=(0, 15), h=0.3)),
    (512, dict(p=(1, 36), alpha=(15, 15), beta=(15, 15), h=1.1)),
]


@pytest.mark.parametrize("n,kw", NIB)
@pytest.mark.parametrize("move,pert", [("pert_fy", 4), ("pert_fy", 3), ("swap", 2), ("window", 4), ("insert", 4)])
def test_nibble_layout_trace_parity(lib, n, kw, move, pert):
    inst = gen.ranged_instance(n, 5, **kw)
    chains, steps, seed = 48, 150, 77 + n
    ins, res, (pen, perm, gid), pr, p, T0 = _run_both(lib, inst, "cdd", chains, steps, seed, samples=300,
                                                     move=move, pert=pert, lanes=8)
    assert lib.sa_layout(ins, chains, lanes=8) == (8, 128 if n > 512 else 64) and ins.query()["small_weights"]
    tr = res["trace"].cpu().numpy()
    for c in range(chains):
        ref = oracle.sa_chain(pr, p, T0, c, trace=True)
        assert np.array_equal(tr[c] >> 1, ref["E_new"]), c
        assert np.array_equal((tr[c] & 1).astype(bool), ref["accepted"]), c
    full = oracle.sa_run(pr, p, T0)
    assert (pen, gid) == (full["E_best"], full["g"]) and np.array_equal(perm, full["best"])
    os.environ["CDD_SA_NO_NIB"] = "1"
    try:
        res2 = lib.sa_run(lib.Instance.from_gen(inst), chains, steps, T0=T0, pert=pert, move=move,
                          seed=seed, trace=True, lanes=8)
    finally:
        del os.environ["CDD_SA_NO_NIB"]
    assert np.array_equal(res2["trace"].cpu().numpy(), tr)


def test_nibble_layout_full_grid_and_balanced(lib):
    # many chains (G = 8 by the automatic layout): every chain's best and final penalty against
    # the oracle, round robin over more chains than resident slots and the balanced schedule
    import torch

    for n, chain_counts in ((1000, (70000, 73040)), (500, (16208, 30000))):
        _full_grid(lib, torch, n, chain_counts)


def _full_grid(lib, torch, n, chain_counts):
    inst = gen.cdd_instance(n, 3, 0.6)
    pr = _prob(inst)
    for chains in chain_counts:
        ins = lib.Instance.from_gen(inst)
        res = lib.sa_run(ins, chains, 40, T0=500.0, seed=11, chain_best=True, chain_final=True)
        torch.cuda.synchronize()
        assert lib.sa_layout(ins, chains) == (8, 128 if n > 512 else 64)
        cb, cf = res["chain_best"].cpu().numpy(), res["chain_final"].cpu().numpy()
        p = oracle.sa_params(chains=1, steps=40, seed=11)
        for c in list(range(0, chains, 997)) + [chains - 1]:
            ref = oracle.sa_chain(pr, p, 500.0, c)
            assert (cb[c], cf[c]) == (ref["E_best"], ref["E_final"]), c


def test_small_weights_flag(lib):
    # cdd_instance_query bit4 follows the layout's conditions (alpha, beta <= 15, pmax * 15 * 120 < 2^16)
    for kw, want in [(dict(p=(1, 20), alpha=(1, 10), beta=(1, 15)), True),
                     (dict(p=(36, 36), alpha=(15, 15), beta=(1, 1)), True),
                     (dict(p=(37, 37), alpha=(15, 15), beta=(1, 1)), False),
                     (dict(p=(1, 20), alpha=(1, 16), beta=(1, 15)), False),
                     (dict(p=(1, 20), alpha=(1, 10), beta=(1, 16)), False)]:
        inst = gen.ranged_instance(600, 2, h=0.5, **kw)
        assert lib.Instance.from_gen(inst).query()["small_weights"] == want, kw
