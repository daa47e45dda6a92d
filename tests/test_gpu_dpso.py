"""GPU parity: DPSO (Alg. 2, eq. (3)) replayed against the oracle (bit-exact swarm-best traces)."""
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


@pytest.mark.parametrize("n,particles,iters,problem,w,c1,c2", [
    (10, 64, 50, "cdd", 0.5, 0.5, 0.5),
    (37, 100, 40, "cdd", 0.3, 0.7, 0.9),
    (100, 256, 30, "cdd", 0.5, 0.5, 0.5),
    (200, 96, 20, "ucddcp", 0.5, 0.5, 0.5),
    (500, 64, 10, "cdd", 1.0, 1.0, 1.0),
    (1000, 40, 6, "cdd", 0.5, 0.5, 0.5),
    (60, 50, 20, "cdd", 0.0, 0.0, 0.0),
])
def test_dpso_parity(lib, n, particles, iters, problem, w, c1, c2):
    import torch

    inst = gen.ucddcp_instance(n, 2) if problem == "ucddcp" else gen.cdd_instance(n, 3, 0.6)
    ins = lib.Instance.from_gen(inst)
    seed = 4321 + n
    res = lib.dpso_run(ins, particles, iters, problem=problem, w=w, c1=c1, c2=c2, seed=seed,
                       trace=True)
    torch.cuda.synchronize()
    pen, perm, gid = lib.best_get(ins)
    pr = oracle.Problem.from_instance(inst)
    P = oracle.CDD if problem == "cdd" else oracle.UCDDCP
    ref = oracle.dpso_run(pr, oracle.dpso_params(problem=P, particles=particles, iters=iters, w=w,
                                                 c1=c1, c2=c2, seed=seed), trace=True)
    assert np.array_equal(res["gbest_trace"].cpu().numpy()[:iters], ref["gbest_trace"])
    assert (pen, gid) == (ref["E_best"], ref["id"])
    assert np.array_equal(perm, ref["best"])


def test_dpso_emulated_two_ranks(lib):
    # the stepping interface with a host-side exchange reproduces the single swarm of 2P particles
    import torch

    inst = gen.cdd_instance(80, 4, 0.4)
    P, iters, seed = 48, 12, 99
    ranks = []
    for r in range(2):
        ins = lib.Instance.from_gen(inst)
        ranks.append((ins, lib.Dpso(ins, P, iters, seed=seed, particle_offset=r * P, trace=True)))
    for ins, sw in ranks:
        sw.begin()

    def exchange(t):
        torch.cuda.synchronize()
        views = [sw.gbest_tensors(t) for _, sw in ranks]
        keys = [int(k.item()) for k, _ in views]
        kmin = min(keys)
        owner = (kmin & 0xFFFFFFFF) // P
        win = views[owner][1].clone()
        for k, p in views:
            k.fill_(kmin)
            p.copy_(win)
        torch.cuda.synchronize()

    for t in range(iters):
        exchange(t)
        for _, sw in ranks:
            sw.iterate(t)
    exchange(iters)
    for _, sw in ranks:
        sw.end()
    torch.cuda.synchronize()
    pr = oracle.Problem.from_instance(inst)
    ref = oracle.dpso_run(pr, oracle.dpso_params(particles=2 * P, iters=iters, seed=seed), trace=True)
    for ins, sw in ranks:
        pen, perm, gid = lib.best_get(ins)
        assert (pen, gid) == (ref["E_best"], ref["id"]) and np.array_equal(perm, ref["best"])
        assert np.array_equal(sw.trace.cpu().numpy(), ref["gbest_trace"])


def test_dpso_n10_reaches_optimum(lib):
    import json
    import os

    gold = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "config1.json")))
    inst = gen.cdd_instance(10, 1, 0.4)
    ins = lib.Instance.from_gen(inst)
    lib.dpso_run(ins, 768, 200, seed=5)  # 768 particles as in the paper
    pen, perm, gid = lib.best_get(ins)
    assert pen == gold["optimum"]


def test_peer_exchange_api_single_rank(lib):
    # the fused-exchange entry points on one rank: argument / state errors, and a world-1 exchange
    # (no peers) equals dpso_run and sa_sync_run exactly
    import torch

    inst = gen.cdd_instance(120, 4, 0.4)
    ins = lib.Instance.from_gen(inst)
    sw = lib.Dpso(ins, 96, 12, seed=5, trace=True)
    with pytest.raises(lib.CddError) as e:
        sw.run_peer()  # no exchange yet
    assert e.value.code == lib.CDD_ESTATE
    with pytest.raises(lib.CddError) as e:
        lib.dpso_peer_create(ins, 2, 2)  # rank outside [0, world)
    assert e.value.code == lib.CDD_EINVAL
    h = lib.dpso_peer_create(ins, 1, 0)
    assert len(h) == lib.IPC_HANDLE_BYTES
    with pytest.raises(lib.CddError) as e:
        lib.dpso_peer_create(ins, 1, 0)  # one exchange per instance
    assert e.value.code == lib.CDD_ESTATE
    with pytest.raises(lib.CddError) as e:
        sw.run_peer()  # created, not open
    assert e.value.code == lib.CDD_ESTATE
    lib.dpso_peer_open(ins, [h])
    lib.dpso_peer_reset(ins)
    sw.run_peer()
    torch.cuda.synchronize()
    got, gtr = lib.best_get(ins), sw.trace.cpu().numpy()
    ref = lib.Instance.from_gen(inst)
    r = lib.dpso_run(ref, 96, 12, seed=5, trace=True)
    torch.cuda.synchronize()
    want = lib.best_get(ref)
    assert got[0] == want[0] and got[2] == want[2] and np.array_equal(got[1], want[1])
    assert np.array_equal(gtr, r["gbest_trace"].cpu().numpy())
    bad = lib.Dpso(ins, 96, 12, seed=5, particle_offset=7)
    with pytest.raises(lib.CddError) as e:
        bad.run_peer()  # particle_offset must be rank * particles
    assert e.value.code == lib.CDD_EINVAL
    with pytest.raises(lib.CddError) as e:
        sw.run_peer()  # a second fused run without dpso_peer_reset
    assert e.value.code == lib.CDD_ESTATE
    # synchronous SA through the same exchange
    lib.dpso_peer_reset(ins)
    ss = lib.SaSync(ins, 2048, 6, 4, seed=9, t0_samples=300).run_peer()
    torch.cuda.synchronize()
    s_ref = lib.SaSync(ref, 2048, 6, 4, seed=9, t0_samples=300).run()
    torch.cuda.synchronize()
    assert lib.best_get(ins)[0] == lib.best_get(ref)[0]
    assert np.array_equal(ss.level_min.cpu().numpy(), s_ref.level_min.cpu().numpy())
    lib.dpso_peer_destroy(ins)
    with pytest.raises(lib.CddError):
        sw.run_peer()
    ins.destroy()
    ref.destroy()


def test_config4_full_size_parity(lib):
    # BASELINE config 4 exactly as bench.py launches it (CDD n=500, h=0.6, instance seed 1, 8192
    # particles x 200 iterations, seed 0x5EED0004, one persistent launch): the oracle replays the
    # whole swarm (~10 s) -- best value, particle id, sequence and the per-iteration swarm best
    import torch

    inst = gen.cdd_instance(500, 1, 0.6)
    ins = lib.Instance.from_gen(inst)
    sw = lib.Dpso(ins, 8192, 200, seed=0x5EED0004, trace=True).run()
    torch.cuda.synchronize()
    got = lib.best_get(ins)
    ref = oracle.dpso_run(oracle.Problem.from_instance(inst),
                          oracle.dpso_params(particles=8192, iters=200, seed=0x5EED0004), trace=True)
    assert (got[0], got[2]) == (ref["E_best"], ref["id"])
    assert np.array_equal(got[1], ref["best"])
    assert np.array_equal(sw.trace.cpu().numpy(), ref["gbest_trace"])


@pytest.mark.parametrize("kernel", ["warp", "group"])
@pytest.mark.parametrize("n,particles,iters,problem", [(37, 100, 25, "cdd"), (300, 64, 10, "ucddcp"),
                                                      (1000, 40, 6, "cdd")])
def test_dpso_both_kernels(lib, monkeypatch, kernel, n, particles, iters, problem):
    # the warp-per-particle and the group-layout iteration kernels are both bit-exact (the library
    # picks by n; CDD_DPSO forces one)
    import torch

    monkeypatch.setenv("CDD_DPSO", kernel)
    inst = gen.ucddcp_instance(n, 5) if problem == "ucddcp" else gen.cdd_instance(n, 4, 0.4)
    ins = lib.Instance.from_gen(inst)
    res = lib.dpso_run(ins, particles, iters, problem=problem, seed=77 + n, trace=True)
    torch.cuda.synchronize()
    pen, perm, gid = lib.best_get(ins)
    P = oracle.CDD if problem == "cdd" else oracle.UCDDCP
    ref = oracle.dpso_run(oracle.Problem.from_instance(inst),
                          oracle.dpso_params(problem=P, particles=particles, iters=iters, seed=77 + n), trace=True)
    assert np.array_equal(res["gbest_trace"].cpu().numpy()[:iters], ref["gbest_trace"])
    assert (pen, gid) == (ref["E_best"], ref["id"]) and np.array_equal(perm, ref["best"])


def test_dpso_more_particles_than_slots(lib):
    # more particles than resident slots (n = 300: ~8200 slots on a B200): every CTA runs several
    # batches per iteration, so the single-GPU publish must map a key's particle to the CTA that
    # holds it across batches (slot rows by parity), and the swarm-best trace must still match
    import torch

    inst = gen.cdd_instance(300, 6, 0.6)
    ins = lib.Instance.from_gen(inst)
    P, iters, seed = 9001, 4, 0x5107
    res = lib.dpso_run(ins, P, iters, seed=seed, trace=True)
    torch.cuda.synchronize()
    pen, perm, gid = lib.best_get(ins)
    ref = oracle.dpso_run(oracle.Problem.from_instance(inst),
                          oracle.dpso_params(particles=P, iters=iters, seed=seed), trace=True)
    assert np.array_equal(res["gbest_trace"].cpu().numpy()[:iters], ref["gbest_trace"])
    assert (pen, gid) == (ref["E_best"], ref["id"]) and np.array_equal(perm, ref["best"])
