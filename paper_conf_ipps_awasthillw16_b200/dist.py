"""Multi-GPU reduction of the best sequence (one process per GPU, torch.distributed).

Asynchronous SA shards naturally: rank r runs global chain ids [r*C, (r+1)*C) with identical
per-chain Philox streams, so the result does not depend on the number of GPUs.  The
only exchange is the final reduction of P:226-228 lifted across GPUs: a MIN all-reduce of the packed
int64 key (penalty << 32 | global chain id) in place on the library's device buffer, then a
broadcast of the winner's int16 sequence (as uint8: NCCL has no int16) from the owning rank.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

from . import best_device_tensors


def owner_rank(key: int, ids_per_rank: int) -> int:
    """Rank that owns the global id packed in `key` (ids are rank-contiguous)."""
    return int(key & 0xFFFFFFFF) // int(ids_per_rank)


# The library's keys are unsigned 64-bit (penalty << 32 | id) with the empty key 0xFFFF...FFFF; the
# collectives see them as signed int64.  Valid keys are < 2^63 (penalties < 2^31), so only the empty
# key (-1 when signed) must be lifted to INT64_MAX before a MIN and restored afterwards.
_EMPTY_SIGNED = -1
_INT64_MAX = (1 << 63) - 1


def _lift_empty(key: torch.Tensor) -> None:
    key.masked_fill_(key == _EMPTY_SIGNED, _INT64_MAX)


def _restore_empty(key: torch.Tensor) -> None:
    key.masked_fill_(key == _INT64_MAX, _EMPTY_SIGNED)


def reduce_best(key: torch.Tensor, perm: torch.Tensor, ids_per_rank: int, group=None) -> int:
    """In place: key <- MIN over ranks; perm <- the winner's perm.  Returns the winner's rank
    (-1 if no rank holds a result; key and perm are then left empty / unchanged).

    `key` is an int64 [1] tensor, `perm` an int16 [n] tensor (device tensors with NCCL, CPU tensors
    with gloo).  One all-reduce and one broadcast; the broadcast source is known to every rank
    from the reduced key.  Raises if the owner computed from the key is not a rank that holds it
    (two ranks with overlapping id ranges, or a wrong ids_per_rank)."""
    local = key.clone()
    _lift_empty(key)
    dist.all_reduce(key, op=dist.ReduceOp.MIN, group=group)
    k = int(key.item())
    if k == _INT64_MAX:
        _restore_empty(key)
        return -1
    src = owner_rank(k, ids_per_rank)
    if not 0 <= src < dist.get_world_size(group):
        raise RuntimeError(f"best key {k:#x}: owner rank {src} outside the world")
    hit = torch.tensor([1 if int(local.item()) == k else 0], dtype=torch.int64, device=key.device)
    dist.all_reduce(hit, op=dist.ReduceOp.SUM, group=group)
    if int(hit.item()) != 1:
        raise RuntimeError(f"best key {k:#x} held by {int(hit.item())} ranks (ids must be disjoint)")
    dist.broadcast(perm.view(torch.uint8), src=src, group=group)
    return src


def reduce_best_async(key: torch.Tensor, perm: torch.Tensor, group=None) -> None:
    """Same result as reduce_best without a host round trip (nothing is read back): the key is
    MIN-all-reduced, every rank but the owner (whose local key equals the minimum -- keys are
    unique, they carry the global id) zeroes its sequence, and the sequences are SUM-all-reduced as
    bytes, which leaves exactly the owner's.  Two collectives queued on the stream, so a loop of
    exchanges (DPSO iterations, synchronous-SA levels) never waits on the host.  Ranks without a
    result (empty key) never win; if no rank has one the key stays empty and the sequences sum to
    zero.  Uniqueness of the winner is the caller's contract (disjoint id ranges); reduce_best
    checks it."""
    local = key.clone()
    _lift_empty(key)
    dist.all_reduce(key, op=dist.ReduceOp.MIN, group=group)
    perm.mul_(((local == key) & (key != _INT64_MAX)).to(perm.dtype))
    _restore_empty(key)
    dist.all_reduce(perm.view(torch.uint8), op=dist.ReduceOp.SUM, group=group)


def reduce_best_wide(pen_id: torch.Tensor, perm: torch.Tensor, group=None) -> None:
    """Generic-path instances (penalties beyond the packed key): pen_id = int64 [2] {penalty, global
    id}, empty = {-1, -1}.  In place: the lexicographic minimum over ranks and the owner's sequence
    -- MIN of the penalty, MIN of the id among the ranks holding it, then a SUM of the sequences
    with every non-owner's zeroed (no host round trip)."""
    pen, gid = pen_id[0:1].clone(), pen_id[1:2].clone()
    empty = pen < 0
    pen.masked_fill_(empty, _INT64_MAX)
    p = pen.clone()
    dist.all_reduce(p, op=dist.ReduceOp.MIN, group=group)
    g = torch.where((pen == p) & ~empty, gid, torch.full_like(gid, _INT64_MAX))
    dist.all_reduce(g, op=dist.ReduceOp.MIN, group=group)
    mine = (pen == p) & (gid == g) & ~empty
    perm.mul_(mine.to(perm.dtype))
    dist.all_reduce(perm.view(torch.uint8), op=dist.ReduceOp.SUM, group=group)
    none = p == _INT64_MAX
    pen_id[0:1].copy_(torch.where(none, torch.full_like(p, -1), p))
    pen_id[1:2].copy_(torch.where(none, torch.full_like(g, -1), g))


def global_best(inst, ids_per_rank: int, group=None) -> int:
    """Reduce the instance's device-resident best (after sa_run / dpso_run) across all ranks.
    Returns the owner's rank (fast path; -1 without a result; generic path: -2, not computed)."""
    if getattr(inst, "wide", False):
        from . import best_device_tensors_wide

        pen_id, perm = best_device_tensors_wide(inst)
        reduce_best_wide(pen_id, perm, group)
        return -2
    key, perm = best_device_tensors(inst)
    return reduce_best(key, perm, ids_per_rank, group)


def global_best_async(inst, group=None) -> None:
    """global_best without the host round trip (reduce_best_async on the best buffers): the next
    run's launches queue behind the collectives instead of waiting for them."""
    if getattr(inst, "wide", False):
        from . import best_device_tensors_wide

        pen_id, perm = best_device_tensors_wide(inst)
        reduce_best_wide(pen_id, perm, group)
        return
    key, perm = best_device_tensors(inst)
    reduce_best_async(key, perm, group)


def peer_exchange_open(inst, group=None):
    """Create this rank's DPSO exchange region, all-gather the CUDA IPC handles over the process
    group and map every peer's region (dpso_peer_create / dpso_peer_open)."""
    from . import dpso_peer_create, dpso_peer_open

    world, rank = dist.get_world_size(group), dist.get_rank(group)
    mine = dpso_peer_create(inst, world, rank)
    handles = [None] * world
    dist.all_gather_object(handles, mine, group=group)
    dpso_peer_open(inst, handles)


def dpso_run_distributed(inst, particles_per_rank: int, iters: int, problem="cdd", w=0.5, c1=0.5,
                         c2=0.5, seed=0, group=None, trace=False, exchange="nccl"):
    """One swarm spread over all ranks (global particle ids rank*P .. rank*P+P-1).  The swarm best of
    Alg. 2 line 5 is global every iteration.

    exchange="nccl": after each device-local step the packed key is MIN-all-reduced and the
    winner's sequence delivered to every rank (reduce_best_async: no host round trip, so the
    iterations queue back to back), then iteration t runs.
    exchange="p2p": one launch per rank for the whole run; the exchange happens inside the kernels
    over peer memory (dpso_run_peer; the instance must have been through peer_exchange_open)."""
    from . import Dpso, dpso_peer_reset

    rank = dist.get_rank(group)
    sw = Dpso(inst, particles_per_rank, iters, problem, w, c1, c2, seed,
              particle_offset=rank * particles_per_rank, trace=trace)
    if exchange == "p2p":
        dpso_peer_reset(inst)
        torch.cuda.synchronize(inst.device)
        dist.barrier(group)  # every region re-armed before any rank's kernels start
        sw.run_peer()
        return sw
    sw.begin()
    for t in range(iters):
        key, perm = sw.gbest_tensors(t)
        reduce_best_async(key, perm, group)
        sw.iterate(t)
    key, perm = sw.gbest_tensors(iters)
    reduce_best_async(key, perm, group)
    sw.end()
    return sw


def sa_sync_run_distributed(inst, chains_per_rank: int, markov_len: int, levels: int, group=None,
                            exchange="nccl", **kw):
    """Synchronous SA over all ranks (global chain ids rank*C .. rank*C+C-1): after
    every temperature level the minimal final state is global -- exchange="nccl": its packed key
    is MIN-all-reduced and the state broadcast from its owner before the next level; "p2p": the
    level's finalisation kernel exchanges it over peer memory (sa_sync_run_peer; the instance must
    have been through peer_exchange_open).  The best-ever state is reduced once at the end
    (global_best)."""
    from . import SaSync, dpso_peer_reset

    rank = dist.get_rank(group)
    ss = SaSync(inst, chains_per_rank, markov_len, levels, chain_offset=rank * chains_per_rank, **kw)
    if exchange == "p2p":
        dpso_peer_reset(inst)
        torch.cuda.synchronize(inst.device)
        dist.barrier(group)
        ss.run_peer()
        global_best(inst, chains_per_rank, group)
        return ss
    for j in range(levels):
        ss.level(j)
        key, perm = ss.exchange_tensors()
        reduce_best_async(key, perm, group)
    global_best(inst, chains_per_rank, group)
    return ss
