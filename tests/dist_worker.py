"""Multi-process check of the cross-GPU paths on real kernels (test infrastructure, run by
tests/test_gpu_dist.py under torchrun; with CDD_DIST_BACKEND=gloo several ranks may share one GPU).
Every result is compared with the CPU ORACLE run over all ranks' chains / particles at once:

  * asynchronous SA sharded over ranks + dist.global_best(_async)  ==  oracle.sa_run of all chains
    (penalty, chain id, sequence);
  * dist.dpso_run_distributed (per-iteration swarm-best exchange, NCCL/gloo between launches and
    fused into the kernels over peer memory)  ==  oracle.dpso_run of the whole swarm (best, id,
    sequence, swarm-best trace);
  * dist.sa_sync_run_distributed (per-level exchange, collectives or fused)  ==  oracle.sa_sync of
    all chains (best penalty, chain id, sequence; every level's minimum).

python -m torch.distributed.run --nproc-per-node 2 --master-addr 127.0.0.1 tests/dist_worker.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import gen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_awasthillw16_b200 as cdd  # noqa: E402
from paper_conf_ipps_awasthillw16_b200 import dist as cdist  # noqa: E402


def main():
    backend = os.environ.get("CDD_DIST_BACKEND", "nccl")
    local = int(os.environ.get("LOCAL_RANK", "0")) % torch.cuda.device_count()
    torch.cuda.set_device(local)
    if backend == "nccl":
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    else:
        dist.init_process_group(backend)
    rank, world = dist.get_rank(), dist.get_world_size()
    inst = gen.cdd_instance(200, 3, 0.6)
    pr = oracle.Problem.from_instance(inst)

    def same(got, E, g, J, what):
        assert got[0] == E and got[2] == g and np.array_equal(got[1], J), (what, got, E, g)

    # asynchronous SA: shards + one reduction
    C, steps = 300, 150
    T0 = oracle.t0(pr, oracle.CDD, 21, 500)
    o = oracle.sa_run(pr, oracle.sa_params(chains=world * C, steps=steps, seed=21), T0)
    ins = cdd.Instance.from_gen(inst, device=local)
    cdd.sa_run(ins, C, steps, seed=21, t0_samples=500, chain_offset=rank * C)
    cdist.global_best(ins, C)
    same(cdd.best_get(ins), o["E_best"], o["g"], o["best"], "sa")
    ins = cdd.Instance.from_gen(inst, device=local)  # the same without a host round trip
    cdd.sa_run(ins, C, steps, seed=21, t0_samples=500, chain_offset=rank * C)
    cdist.global_best_async(ins)
    same(cdd.best_get(ins), o["E_best"], o["g"], o["best"], "sa async")

    # DPSO: one swarm over all ranks, exchange every iteration
    P, iters = 48, 25
    o = oracle.dpso_run(pr, oracle.dpso_params(particles=world * P, iters=iters, seed=22), trace=True)
    ins = cdd.Instance.from_gen(inst, device=local)
    sw = cdist.dpso_run_distributed(ins, P, iters, seed=22, trace=True)
    torch.cuda.synchronize()
    same(cdd.best_get(ins), o["E_best"], o["id"], o["best"], "dpso")
    assert np.array_equal(sw.trace.cpu().numpy()[:iters], o["gbest_trace"]), "dpso trace"

    # DPSO with the exchange fused into the kernels over peer memory (CUDA IPC regions; on one
    # GPU the ranks' kernels are time-sliced, which is slow but exercises the same protocol)
    if os.environ.get("CDD_DIST_P2P", "1") == "1":
        ins = cdd.Instance.from_gen(inst, device=local)
        cdist.peer_exchange_open(ins)
        for rep in range(2):  # the region is re-armed per run
            sw = cdist.dpso_run_distributed(ins, P, iters, seed=22, trace=True, exchange="p2p")
            torch.cuda.synchronize()
            same(cdd.best_get(ins), o["E_best"], o["id"], o["best"], f"dpso p2p {rep}")
            assert np.array_equal(sw.trace.cpu().numpy()[:iters], o["gbest_trace"]), "p2p trace"
        # a fused run without re-arming the region is refused
        try:
            sw.run_peer()
            raise AssertionError("run_peer without dpso_peer_reset was accepted")
        except cdd.CddError as e:
            assert e.code == cdd.CDD_ESTATE

    # synchronous SA: exchange of s^min every level
    C, M, L = 96, 10, 12
    T0 = oracle.t0(pr, oracle.CDD, 23, 500)
    o = oracle.sa_sync(pr, oracle.sa_params(chains=world * C, steps=M, seed=23), T0, L)
    ins = cdd.Instance.from_gen(inst, device=local)
    ss = cdist.sa_sync_run_distributed(ins, C, M, L, seed=23, t0_samples=500)
    torch.cuda.synchronize()
    same(cdd.best_get(ins), o["E_best"], o["g"], o["best"], "sync")
    if os.environ.get("CDD_DIST_P2P", "1") == "1":  # the level exchange fused over peer memory
        ins = cdd.Instance.from_gen(inst, device=local)
        cdist.peer_exchange_open(ins)
        ss = cdist.sa_sync_run_distributed(ins, C, M, L, seed=23, t0_samples=500, exchange="p2p")
        torch.cuda.synchronize()
        same(cdd.best_get(ins), o["E_best"], o["g"], o["best"], "sync p2p")
        # every level's s^min is the global one: the level minima equal the oracle's
        assert np.array_equal(ss.level_min.cpu().numpy(), o["level_min_E"]), "sync p2p levels"

    dist.barrier()
    if rank == 0:
        print(f"dist_check ok: world {world}, backend {backend}", flush=True)
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
