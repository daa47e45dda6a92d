"""World-size-2 CPU (gloo) test of the cross-GPU reduction logic (SURVEY T10 sharding invariance).

Each rank runs its shard of SA chains (global ids rank*C .. rank*C+C-1) with the oracle, packs its
local best as (penalty << 32 | global chain id), and calls the same reduce_best() the GPU path uses
over NCCL.  The reduced result must equal one run over all 2C chains."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, C, q):
    import sys

    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import gen
    import oracle
    from paper_conf_ipps_awasthillw16_b200.dist import reduce_best

    inst = gen.cdd_instance(40, 3, 0.4)
    pr = oracle.Problem.from_instance(inst)
    T0 = oracle.t0(pr, oracle.CDD, 5, 300)
    p = oracle.sa_params(chains=C, steps=150, seed=5, chain_offset=rank * C)
    r = oracle.sa_run(pr, p, T0)
    key = torch.tensor([(r["E_best"] << 32) | r["g"]], dtype=torch.int64)
    perm = torch.from_numpy(r["best"].copy())
    src = reduce_best(key, perm, C)
    q.put((rank, int(key.item()), perm.numpy().tolist(), src))
    dist.destroy_process_group()


def test_reduce_best_matches_single_run():
    world, C = 2, 12
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, C, q)) for r in range(world)]
    [p.start() for p in ps]
    res = [q.get(timeout=120) for _ in range(world)]
    [p.join(timeout=60) for p in ps]
    assert all(p.exitcode == 0 for p in ps)
    import gen
    import oracle

    inst = gen.cdd_instance(40, 3, 0.4)
    pr = oracle.Problem.from_instance(inst)
    T0 = oracle.t0(pr, oracle.CDD, 5, 300)
    full = oracle.sa_run(pr, oracle.sa_params(chains=world * C, steps=150, seed=5), T0)
    for rank, key, perm, src in res:
        assert key >> 32 == full["E_best"] and key & 0xFFFFFFFF == full["g"]
        assert perm == full["best"].tolist()
        assert src == full["g"] // C


def test_owner_rank():
    from paper_conf_ipps_awasthillw16_b200.dist import owner_rank

    assert owner_rank((123 << 32) | 70000, 65536) == 1
    assert owner_rank((5 << 32) | 0, 65536) == 0


def _worker_async(rank, world, port, q):
    import sys

    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_awasthillw16_b200.dist import reduce_best, reduce_best_async

    out = []
    rng = np.random.default_rng(100 + rank)
    for trial in range(5):
        # penalties collide across ranks on purpose: the global id in the low word breaks ties
        pen = int(rng.integers(0, 3))
        gid = rank * 1000 + int(rng.integers(0, 1000))
        perm = torch.from_numpy(rng.permutation(37).astype(np.int16))
        k1 = torch.tensor([(pen << 32) | gid], dtype=torch.int64)
        k2 = k1.clone()
        p1, p2 = perm.clone(), perm.clone()
        reduce_best(k1, p1, 1000)
        reduce_best_async(k2, p2)
        out.append((int(k1.item()), int(k2.item()), p1.tolist(), p2.tolist()))
    q.put((rank, out))
    dist.destroy_process_group()


def test_reduce_best_async_equals_broadcast_version():
    world = 3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker_async, args=(r, world, port, q)) for r in range(world)]
    [p.start() for p in ps]
    res = dict(q.get(timeout=120) for _ in range(world))
    [p.join(timeout=60) for p in ps]
    assert all(p.exitcode == 0 for p in ps)
    for trial in range(5):
        rows = [res[r][trial] for r in range(world)]
        k1, k2, p1, p2 = rows[0]
        assert k1 == k2 and p1 == p2
        assert all(r == rows[0] for r in rows)  # every rank holds the same winner


def _worker_empty(rank, world, port, q):
    import sys

    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_awasthillw16_b200.dist import reduce_best, reduce_best_async

    out = []
    perm = torch.full((11,), rank + 1, dtype=torch.int16)
    # (a) rank 1 has no result (empty key 0xFFFF...FFFF = -1 signed): rank 0 / 2 must win
    key = (5 << 32) | (rank * 10) if rank != 1 else -1
    for fn in (reduce_best, reduce_best_async):
        k = torch.tensor([key], dtype=torch.int64)
        p = perm.clone()
        fn(k, p, 10) if fn is reduce_best else fn(k, p)
        out.append((int(k.item()), p.tolist()))
    # (b) nobody has a result: the key stays empty
    k = torch.tensor([-1], dtype=torch.int64)
    src = reduce_best(k, perm.clone(), 10)
    out.append((int(k.item()), src))
    k = torch.tensor([-1], dtype=torch.int64)
    reduce_best_async(k, perm.clone())
    out.append((int(k.item()), None))
    # (c) two ranks claiming the same key (overlapping ids) is detected
    k = torch.tensor([(1 << 32) | 3], dtype=torch.int64)
    try:
        reduce_best(k, perm.clone(), 10)
        out.append("no error")
    except RuntimeError as e:
        out.append("error")
    q.put((rank, out))
    dist.destroy_process_group()


def test_reduce_best_empty_keys_and_collisions():
    # the empty key must never win a signed MIN; a collision must not pass silently
    world = 3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker_empty, args=(r, world, port, q)) for r in range(world)]
    [p.start() for p in ps]
    res = dict(q.get(timeout=120) for _ in range(world))
    [p.join(timeout=60) for p in ps]
    assert all(p.exitcode == 0 for p in ps)
    for r in range(world):
        a, b, c, d, e = res[r]
        assert a == ((5 << 32) | 0, [1] * 11) and b == a
        assert c == (-1, -1) and d == (-1, None)
        assert e == "error"
