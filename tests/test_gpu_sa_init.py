"""GPU parity of asynchronous SA started from caller-given sequences (sa_params.init, "the
initial job sequences are copied to the GPU"): one sequence for every chain, or one per chain,
replayed by the oracle's SA with the same initial sequences."""
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


@pytest.mark.parametrize("n,chains,steps,problem,lanes,shared", [
    (60, 100, 200, "cdd", 0, True),
    (60, 100, 200, "cdd", 32, False),
    (300, 2000, 120, "cdd", 0, False),     # group layout
    (300, 70, 120, "cdd", 8, True),
    (1000, 1200, 60, "cdd", 0, False),    # automatic layout (16 lanes x 64 at 1200 chains)
    (1000, 300, 60, "cdd", 8, False),     # the headline layout: 8 lanes x 128, small-weight records
    (1000, 300, 60, "cdd", 8, True),
    (200, 300, 100, "ucddcp", 0, False),
    (200, 300, 100, "ucddcp", 32, True),
])
def test_sa_from_given_sequences(lib, n, chains, steps, problem, lanes, shared):
    import torch

    inst = gen.ucddcp_instance(n, 4) if problem == "ucddcp" else gen.cdd_instance(n, 4, 0.4)
    ins = lib.Instance.from_gen(inst)
    seed, offset = 31 + n, 5000
    if shared:
        init = gen.random_perms(1, n, 8)[0]
    else:
        init = gen.random_perms(chains, n, 9, ld=n + 5)  # padded rows (init_ld = n + 5)
    res = lib.sa_run(ins, chains, steps, problem=problem, seed=seed, t0_samples=400,
                     chain_offset=offset, trace=True, chain_best=True, lanes=lanes,
                     init=torch.from_numpy(init).cuda())
    torch.cuda.synchronize()
    lib.cdd_check(ins)
    pen, perm, gid = lib.best_get(ins)
    pr = oracle.Problem.from_instance(inst)
    P = oracle.UCDDCP if problem == "ucddcp" else oracle.CDD
    T0 = oracle.t0(pr, P, seed, 400)
    rows = init if shared else init[:, :n]
    p = oracle.sa_params(problem=P, chains=chains, steps=steps, seed=seed, chain_offset=offset,
                         init=rows)
    tr = res["trace"].cpu().numpy()
    cb = res["chain_best"].cpu().numpy()
    for c in list(range(0, chains, max(1, chains // 40))) + [chains - 1]:
        ref = oracle.sa_chain(pr, p, T0, offset + c, trace=True)
        assert np.array_equal(tr[c] >> 1, ref["E_new"]), c
        assert np.array_equal((tr[c] & 1).astype(bool), ref["accepted"]), c
        assert cb[c] == ref["E_best"], c
    full = oracle.sa_run(pr, p, T0)
    assert (pen, gid) == (full["E_best"], full["g"]) and np.array_equal(perm, full["best"])


def test_given_sequence_zero_steps_is_its_penalty(lib):
    # Alg. 1 with no iterations returns s0 itself: its penalty is the batched evaluation's
    import torch

    inst = gen.cdd_instance(500, 6, 0.6)
    ins = lib.Instance.from_gen(inst)
    init = torch.from_numpy(gen.random_perms(1, 500, 3)[0]).cuda()
    lib.sa_run(ins, 10, 0, seed=1, t0_samples=100, init=init)
    torch.cuda.synchronize()
    pen, perm, gid = lib.best_get(ins)
    z = lib.cdd_eval_batch(ins, init[None, :]).item()
    assert pen == z and gid == 0 and np.array_equal(perm, init.cpu().numpy()[:500])


@pytest.mark.parametrize("lanes", [0, 32])
def test_invalid_initial_ids_flagged(lib, lanes):
    import torch

    inst = gen.cdd_instance(100, 2, 0.4)
    ins = lib.Instance.from_gen(inst)
    init = gen.random_perms(64, 100, 5)
    init[17, 40] = 100  # id n
    lib.sa_run(ins, 64, 10, seed=2, t0_samples=100, lanes=lanes, init=torch.from_numpy(init).cuda())
    with pytest.raises(lib.CddError) as e:
        lib.cdd_check(ins)
    assert e.value.code == lib.CDD_EDATA
    lib.cdd_check(ins)  # cleared


def test_given_sequences_under_the_balanced_schedule(lib):
    # caller-given initial sequences and a chain offset with more chains than resident slots and a
    # mostly empty last round: split chains start from their own rows and are resumed from the
    # handover -- every chain's best equals the oracle's replay
    import torch

    n, chains, steps, offset = 120, 15000, 37, 777
    inst = gen.cdd_instance(n, 6, 0.6)
    ins = lib.Instance.from_gen(inst)
    init = gen.random_perms(chains, n, 21, ld=n + 8)
    res = lib.sa_run(ins, chains, steps, seed=41, T0=1800.0, chain_offset=offset, lanes=8,
                     chain_best=True, init=torch.from_numpy(init).cuda())
    torch.cuda.synchronize()
    lib.cdd_check(ins)
    cb = res["chain_best"].cpu().numpy()
    pr = oracle.Problem.from_instance(inst)
    p = oracle.sa_params(chains=chains, steps=steps, seed=41, chain_offset=offset, init=init[:, :n])
    for c in range(chains):
        assert oracle.sa_chain(pr, p, 1800.0, offset + c)["E_best"] == cb[c], c
    pen, perm, gid = lib.best_get(ins)
    assert pen == cb.min() and gid == offset + int(np.argmin(cb))
    assert oracle.cdd_eval(pr, perm) == pen
