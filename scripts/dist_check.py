"""Multi-process check of the cross-GPU paths on real kernels (run under torchrun; with
CDD_DIST_BACKEND=gloo several ranks may share one GPU):

  * asynchronous SA sharded over ranks + dist.global_best  ==  one run of all chains;
  * dist.dpso_run_distributed (per-iteration swarm-best exchange, NCCL/gloo between launches and
    fused into the kernels over peer memory)  ==  one swarm of all particles (best, id, sequence
    and the swarm-best trace);
  * dist.sa_sync_run_distributed (per-level exchange)  ==  one synchronous run of all chains
    (best penalty; R18: the chain holding a tied best may differ).

python -m torch.distributed.run --nproc-per-node 2 --master-addr 127.0.0.1 scripts/dist_check.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import gen  # noqa: E402
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

    # asynchronous SA: shards + one reduction
    C, steps = 300, 150
    ins = cdd.Instance.from_gen(inst, device=local)
    cdd.sa_run(ins, C, steps, seed=21, t0_samples=500, chain_offset=rank * C)
    cdist.global_best(ins, C)
    got = cdd.best_get(ins)
    ref = cdd.Instance.from_gen(inst, device=local)
    cdd.sa_run(ref, world * C, steps, seed=21, t0_samples=500)
    want = cdd.best_get(ref)
    assert got[0] == want[0] and got[2] == want[2] and np.array_equal(got[1], want[1]), ("sa", got, want)
    ins = cdd.Instance.from_gen(inst, device=local)  # the same without a host round trip
    cdd.sa_run(ins, C, steps, seed=21, t0_samples=500, chain_offset=rank * C)
    cdist.global_best_async(ins)
    got = cdd.best_get(ins)
    assert got[0] == want[0] and got[2] == want[2] and np.array_equal(got[1], want[1]), ("sa async", got, want)

    # DPSO: one swarm over all ranks, exchange every iteration
    P, iters = 48, 25
    ins = cdd.Instance.from_gen(inst, device=local)
    sw = cdist.dpso_run_distributed(ins, P, iters, seed=22, trace=True)
    torch.cuda.synchronize()
    got = cdd.best_get(ins)
    ref = cdd.Instance.from_gen(inst, device=local)
    r = cdd.dpso_run(ref, world * P, iters, seed=22, trace=True)
    torch.cuda.synchronize()
    want = cdd.best_get(ref)
    assert got[0] == want[0] and got[2] == want[2] and np.array_equal(got[1], want[1]), ("dpso", got, want)
    assert np.array_equal(sw.trace.cpu().numpy()[:iters], r["gbest_trace"].cpu().numpy()[:iters]), "dpso trace"

    # DPSO with the exchange fused into the kernels over peer memory (CUDA IPC regions; on one
    # GPU the ranks' kernels are time-sliced, which is slow but exercises the same protocol)
    if os.environ.get("CDD_DIST_P2P", "1") == "1":
        ins = cdd.Instance.from_gen(inst, device=local)
        cdist.peer_exchange_open(ins)
        for rep in range(2):  # the region is re-armed per run
            sw = cdist.dpso_run_distributed(ins, P, iters, seed=22, trace=True, exchange="p2p")
            torch.cuda.synchronize()
            got = cdd.best_get(ins)
            assert got[0] == want[0] and got[2] == want[2] and np.array_equal(got[1], want[1]), ("p2p", rep, got, want)
            assert np.array_equal(sw.trace.cpu().numpy()[:iters], r["gbest_trace"].cpu().numpy()[:iters]), "p2p trace"

    # synchronous SA: exchange of s^min every level
    C, M, L = 96, 10, 12
    ins = cdd.Instance.from_gen(inst, device=local)
    cdist.sa_sync_run_distributed(ins, C, M, L, seed=23, t0_samples=500)
    torch.cuda.synchronize()
    got = cdd.best_get(ins)
    ref = cdd.Instance.from_gen(inst, device=local)
    ref_ss = cdd.SaSync(ref, world * C, M, L, seed=23, t0_samples=500).run()
    torch.cuda.synchronize()
    want = cdd.best_get(ref)
    assert got[0] == want[0], ("sync", got[0], want[0])
    if os.environ.get("CDD_DIST_P2P", "1") == "1":  # the level exchange fused over peer memory
        ins = cdd.Instance.from_gen(inst, device=local)
        cdist.peer_exchange_open(ins)
        ss = cdist.sa_sync_run_distributed(ins, C, M, L, seed=23, t0_samples=500, exchange="p2p")
        torch.cuda.synchronize()
        got = cdd.best_get(ins)
        assert got[0] == want[0], ("sync p2p", got[0], want[0])
        # every level's s^min is the global one: the level minima equal the single run's
        assert np.array_equal(ss.level_min.cpu().numpy(), ref_ss.level_min.cpu().numpy()), "sync p2p levels"

    dist.barrier()
    if rank == 0:
        print(f"dist_check ok: world {world}, backend {backend}", flush=True)
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
