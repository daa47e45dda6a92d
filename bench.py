"""Benchmark: sequence evaluations/s of the parallel-SA hot path at n=1000 on B200 (BASELINE.json).

One bench "step" = one pass of the whole hot path over BASELINE config 5 on this GPU: for each of
the four CDD n=1000 instances (seed 1, h in {0.2,0.4,0.6,0.8}) the T0 rule (5000 random
sequences), then 65,536 asynchronous SA chains x 5000 iterations (Alg. 1, P:194-198,
mu=0.88, Pert=4 FY moves), then the reduction to the best -- and, on N>1 GPUs, the
NCCL MIN all-reduce of the packed best plus the winner broadcast.  value = all sequence
evaluations of all ranks / max-over-ranks device time.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl reference]
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

N_JOBS = 1000
CHAINS = 65536
SA_STEPS = 5000
T0_SAMPLES = 5000
HS = (0.2, 0.4, 0.6, 0.8)
INSTANCE_SEED = 1
RUN_SEED = 0x5EED0005
METRIC = "sequence evals/s at n=1000 on 1/8 B200; SA % gap vs best-known"
WORKLOAD = ("config5: CDD n=1000, h in {{0.2,0.4,0.6,0.8}} (instance seed 1), {chains} SA chains/GPU x "
            "{steps} steps, T0 from 5000 samples")
INT_OPS_PER_ELEM = 6  # 3 prefix adds + subtract + select + multiply-add per job


_T_START = time.time()


def _log(msg):
    """Progress on stderr (stdout carries only the JSON line)."""
    print(f"[bench {time.time() - _T_START:7.1f}s] {msg}", file=sys.stderr, flush=True)


def _peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


def _int_peak():
    """Best measured integer rate of this GPU model (scripts/int_peak.cu, committed measurements)."""
    best = {"op": "nominal 4 SMSP x 32 lanes", "lane_ops_per_clk_per_sm": 128.0,
            "warp_instr_per_clk_per_sm": 4.0}
    path = os.path.join(ROOT, "profiles", "r2_int_peak.jsonl")
    if os.path.exists(path):
        rows = [json.loads(x) for x in open(path) if x.strip().startswith("{")]
        if rows:
            best = max(rows, key=lambda r: r["lane_ops_per_clk_per_sm"])
    return best


def _evals_per_step(chains, steps, samples, instances):
    return instances * (samples + chains * (steps + 1))


class ClockSampler:
    """nvidia-smi clocks and throttle reasons sampled during the timed region."""

    def __init__(self, index=0):
        self.index = index
        self.proc = None
        self.lines = []

    def __enter__(self):
        q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--id={self.index}", f"--query-gpu={q}", "--format=csv,noheader,nounits",
                 "-lms", "200"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if self.proc is not None:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 8:
                continue
            try:
                sm.append(float(f[0]))
                mx = float(f[1])
            except ValueError:
                continue
            for nm, v in zip(names, f[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------------------ reference arm
def run_reference(args):
    """The CPU oracle (oracle/, untuned) on the box's host cores: a bounded sample of the same
    workload (a few chains x steps of the same instances), same metric and unit."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import gen
    import oracle

    threads = len(os.sched_getaffinity(0)) or os.cpu_count() or 1
    chains_per_thread, steps = 1, 4000  # ~0.1-0.3 s of CPU work per bench step
    insts = [oracle.Problem.from_instance(gen.cdd_instance(N_JOBS, INSTANCE_SEED, h)) for h in HS]
    T0s = [oracle.t0(pr, oracle.CDD, RUN_SEED, 200) for pr in insts]

    def one_step():
        t = time.perf_counter()
        for pr, T0 in zip(insts, T0s):
            def work(tid):
                p = oracle.sa_params(chains=chains_per_thread, steps=steps, seed=RUN_SEED,
                                     chain_offset=tid * chains_per_thread)
                oracle.sa_run(pr, p, T0)
            ts = [threading.Thread(target=work, args=(i,)) for i in range(threads)]
            [x.start() for x in ts]
            [x.join() for x in ts]
        return time.perf_counter() - t

    _log("warmup")
    for _ in range(args.warmup):
        one_step()
    dts = [one_step() for _ in range(args.steps)]
    evals = len(HS) * threads * chains_per_thread * (steps + 1)
    value = evals * args.steps / sum(dts)
    sample = (f"{len(HS)} instances x {threads} threads x {chains_per_thread} chain x {steps} SA "
              f"steps per bench step (T0 from 200 samples, excluded)")
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "evals/s",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1000 * sum(dts) / args.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "config": {"workload": WORKLOAD.format(chains=CHAINS, steps=SA_STEPS), "sample": sample},
            "cpu_baseline": {"value": value, "unit": "evals/s", "cores": threads, "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": value, "unit": "evals/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def _cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def cpu_baseline_sample(seconds=12.0):
    """Oracle SA timed on the host cores (bounded sample of the same workload), plus the oracle's
    single-thread rate and its batched-evaluation rate (BASELINE.md's CPU-baseline plan)."""
    import gen
    import numpy as np
    import oracle

    threads = len(os.sched_getaffinity(0)) or os.cpu_count() or 1
    inst = gen.cdd_instance(N_JOBS, INSTANCE_SEED, 0.4)
    pr = oracle.Problem.from_instance(inst)
    T0 = oracle.t0(pr, oracle.CDD, RUN_SEED, 200)
    # single thread: one chain for ~2 s; sizes the per-thread chain of the all-core sample
    t = time.perf_counter()
    oracle.sa_chain(pr, oracle.sa_params(steps=200, seed=RUN_SEED), T0, 0)
    per_eval = (time.perf_counter() - t) / 201
    st_steps = max(50, int(2.0 / per_eval))
    t = time.perf_counter()
    oracle.sa_chain(pr, oracle.sa_params(steps=st_steps, seed=RUN_SEED), T0, 1)
    single = (st_steps + 1) / (time.perf_counter() - t)
    steps = max(50, int(seconds / per_eval))
    done = [0]

    def work(tid):
        oracle.sa_chain(pr, oracle.sa_params(steps=steps, seed=RUN_SEED), T0, tid)
        done[0] += steps + 1

    ts = [threading.Thread(target=work, args=(i,)) for i in range(threads)]
    t = time.perf_counter()
    [x.start() for x in ts]
    [x.join() for x in ts]
    dt = time.perf_counter() - t
    # batched evaluation (the cdd_eval_batch leg's workload: random sequences at n=1000): one
    # bounded batch (generating the sequences is single-threaded numpy, so its size must not grow
    # with the core count), evaluated on all threads repeatedly for ~3 s
    rows = min(256 * threads, 16384)
    perms = gen.random_perms(rows, N_JOBS, 7, ld=N_JOBS)
    bounds = np.linspace(0, rows, threads + 1).astype(np.int64)
    cnt = [0] * threads

    def ework(tid):
        a, b = int(bounds[tid]), int(bounds[tid + 1])
        t1 = time.perf_counter()
        while b > a and time.perf_counter() - t1 < 3.0:
            oracle.eval_batch(pr, perms[a:b])
            cnt[tid] += b - a

    ts = [threading.Thread(target=ework, args=(i,)) for i in range(threads)]
    t = time.perf_counter()
    [x.start() for x in ts]
    [x.join() for x in ts]
    ev_rate = sum(cnt) / (time.perf_counter() - t)
    reps = sum(cnt) // rows
    return {"value": done[0] / dt, "unit": "evals/s", "cores": threads, "kind": "oracle",
            "cpu_model": _cpu_model(), "single_thread_evals_per_s": single,
            "eval_batch_evals_per_s": ev_rate,
            "sample": f"{threads} host threads x 1 SA chain x {steps} steps, CDD n=1000 h=0.4 "
                      f"(T0 from 200 samples, excluded); {dt:.1f} s; single thread {st_steps} steps; "
                      f"batched evaluation of {rows} random sequences x {reps} passes on {threads} threads"}


# ------------------------------------------------------------------------------ GPU arm
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--chains", type=int, default=CHAINS)
    ap.add_argument("--sa-steps", type=int, default=SA_STEPS)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-eval", action="store_true")
    ap.add_argument("--no-configs", action="store_true")
    ap.add_argument("--no-quality", action="store_true")
    args = ap.parse_args()
    if os.environ.get("CDD_BENCH_WATCHDOG"):  # dump every thread's stack if a phase hangs
        import faulthandler
        faulthandler.dump_traceback_later(int(os.environ["CDD_BENCH_WATCHDOG"]), exit=True)
    if args.impl == "reference":
        return run_reference(args)

    import numpy as np
    import torch
    import torch.distributed as dist

    import gen
    import paper_conf_ipps_awasthillw16_b200 as lib
    from paper_conf_ipps_awasthillw16_b200 import dist as cdist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # CDD_BENCH_DEVICES=k maps local ranks onto k GPUs (test hook: several ranks on one GPU need
    # CDD_BENCH_BACKEND=gloo, NCCL refuses duplicate devices); default one GPU per rank, NCCL
    local = local % int(os.environ.get("CDD_BENCH_DEVICES", str(max(1, torch.cuda.device_count()))))
    torch.cuda.set_device(local)
    if world > 1:
        backend = os.environ.get("CDD_BENCH_BACKEND", "nccl")
        # the communicator log (ranks, devices, transports: NVLink / NVLS) on stderr, so the JSON
        # line stays alone on stdout
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        os.environ.setdefault("NCCL_DEBUG_FILE", "/dev/stderr")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    dev = torch.device("cuda", local)
    stream = torch.cuda.current_stream(dev)

    chains, steps = args.chains, args.sa_steps
    gens = [gen.cdd_instance(N_JOBS, INSTANCE_SEED, h) for h in HS]
    insts = [lib.Instance.from_gen(g, device=local) for g in gens]
    ws = {}
    T0buf = [torch.empty(1, dtype=torch.float64, device=dev) for _ in insts]
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    kernel_ev = []

    def one_step(record=False):
        out = []
        for i, ins in enumerate(insts):
            flush.fill_(i)  # L2 flush between instances (256 MiB write)
            T0 = lib.sa_t0(ins, "cdd", seed=RUN_SEED, samples=T0_SAMPLES)
            e1 = torch.cuda.Event(enable_timing=True)
            e2 = torch.cuda.Event(enable_timing=True)
            e1.record(stream)
            r = lib.sa_run(ins, chains, steps, seed=RUN_SEED, chain_offset=rank * chains,
                           T0_dev=T0, workspace=ws.get(i))
            e2.record(stream)
            ws[i] = r["workspace"]
            if record:
                kernel_ev.append((e1, e2))
            if world > 1:
                cdist.global_best_async(ins)  # no host sync between instances
            out.append(ins)
        return out

    _log("warmup")
    for _ in range(args.warmup):
        one_step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    with ClockSampler(local) as clk:
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        t0 = torch.cuda.Event(enable_timing=True)
        t1 = torch.cuda.Event(enable_timing=True)
        t0.record(stream)
        for _ in range(args.steps):
            one_step(record=True)
        t1.record(stream)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
    ms = t0.elapsed_time(t1)
    if world > 1:
        tt = torch.tensor([ms], device=dev, dtype=torch.float64)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms = float(tt.item())
    evals = _evals_per_step(chains, steps, T0_SAMPLES, len(insts)) * args.steps * world
    value = evals / (ms / 1000.0)

    # quality: best of the last step per instance vs the oracle-made best-known values
    gaps = {}
    bk = _best_known()
    for g, ins in zip(gens, insts):
        pen, perm, gid = lib.best_get(ins)
        key = f"{g.h:.1f}"
        entry = {"best": pen, "chain": gid}
        if g.name() in bk:
            ref = bk[g.name()]["penalty"]
            entry["best_known"] = ref
            entry["gap_pct"] = 100.0 * (pen - ref) / ref
        gaps[key] = entry

    # roofline of the dominant kernel (sa_group_kernel): algorithmic int ops / its event duration,
    # against the MEASURED integer peak of this B200 (scripts/int_peak.cu -> profiles/r2_int_peak.jsonl:
    # the best lane-op rate of the measured opcode mixes), plus the issue view (ncu-counted warp
    # instructions per evaluation / measured best warp-instruction rate)
    peaks = _peaks()
    sm_max = float(peaks.get("sm_max_mhz", 1965.0))
    kms = [a.elapsed_time(b) for a, b in kernel_ev]
    k_avg_ms = sum(kms) / len(kms)
    evals_launch = chains * (steps + 1)
    ops = INT_OPS_PER_ELEM * N_JOBS * evals_launch
    achieved = ops / (k_avg_ms / 1000.0) / 1e12
    nsm = torch.cuda.get_device_properties(dev).multi_processor_count
    ip = _int_peak()
    peak = ip["lane_ops_per_clk_per_sm"] * nsm * sm_max * 1e6 / 1e12
    traffic = None
    tp = os.path.join(ROOT, "profiles", "sa_kernel_dram_bytes.json")
    if os.path.exists(tp):
        traffic = json.load(open(tp)).get("dram_bytes_per_launch")
    step_ms = ms / args.steps
    G, E = lib.sa_layout(insts[0], chains)
    nib = (G, E) == (8, 128) and insts[0].query()["small_weights"] and not os.environ.get("CDD_SA_NO_NIB")
    kname = (f"sa_group_kernel<{G},{E}> (CDD, {32 // G} chains per warp"
             + (", 4-bit weights + sub-block summaries)" if nib else ")") if G < 32
             else f"sa_kernel<{E}> (CDD, one warp per chain)")
    # The bound is instruction issue: the kernel does byte-SIMD (one IMAD forms four byte prefixes,
    # one IDP.4A dots four jobs), so the 6n ALGORITHMIC ops per evaluation can run faster than one
    # int32 lane-op each and their rate is no fraction of the lane-op peak.  achieved = issued
    # lane-ops (ncu-counted warp instructions per evaluation x 32, profiles/sa_kernel_issue.json)
    # per second of the live kernel time; peak = the best measured issue rate (r2_int_peak.jsonl).
    ipath = os.path.join(ROOT, "profiles", "sa_kernel_issue.json")
    ipe = json.load(open(ipath))["warp_instr_per_eval"] if os.path.exists(ipath) else None
    alg = {"ops_per_eval": INT_OPS_PER_ELEM * N_JOBS, "ops_per_launch": ops, "achieved": achieved,
           "unit": "Tint-op/s", "ratio_to_int32_lane_peak": achieved / peak,
           "note": f"{INT_OPS_PER_ELEM}n algorithmic int ops per evaluation (SURVEY 8(d)); byte-SIMD "
                   "packs four of them into one lane-op, and on the small-weight layout a step "
                   "recomputes only the <= 4 changed 16-position sub-blocks (the others' forms are "
                   "cached), so this ratio exceeds 1 -- the issue fraction is the bound"}
    if ipe is not None:
        issued = ipe * 32 * evals_launch / (k_avg_ms / 1000.0) / 1e12
        rate = ipe * evals_launch / (k_avg_ms / 1000.0) / (nsm * sm_max * 1e6)
        roofline = {"bound": "alu", "achieved": issued, "peak": peak, "unit": "Tint-op/s",
                    "frac": issued / peak, "basis": "issued lane-ops (32 x warp instructions)",
                    "warp_instr_per_eval": ipe, "achieved_warp_instr_per_clk_per_sm": rate,
                    "peak_warp_instr_per_clk_per_sm": ip["warp_instr_per_clk_per_sm"]}
    else:
        roofline = {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "Tint-op/s",
                    "frac": achieved / peak, "basis": "algorithmic ops"}
    roofline.update({"traffic": traffic, "kernel": kname, "kernel_ms_avg": k_avg_ms,
                     "kernel_share_of_step": k_avg_ms * len(insts) / step_ms, "algorithmic": alg,
                     "peak_note": (f"measured: {ip['lane_ops_per_clk_per_sm']:.1f} int32 lane-ops/clk/SM "
                                   f"({ip['op']}, scripts/int_peak.cu, profiles/r2_int_peak.jsonl) x {nsm} SMs x "
                                   f"{sm_max:.0f} MHz max clock; instructions per evaluation from ncu "
                                   f"(profiles/sa_kernel_issue.json)")})

    _log("timed region done")
    extra = {}
    _log("eval_batch")
    if rank == 0 and not args.no_eval:
        extra["eval_batch"] = bench_eval(lib, gens[1], dev, stream, peaks)
    _log("other configs")
    if rank == 0 and not args.no_configs:
        extra["other_configs"] = bench_configs(lib, dev, stream)
    _log("quality table")
    if rank == 0 and not args.no_quality:
        extra["quality_table"] = bench_quality(lib, dev, stream)
    if world > 1 and not args.no_configs:
        dm = bench_dpso_multi_gpu(lib, cdist, dev, rank, world)
        if rank == 0:
            extra["dpso_multi_gpu"] = dm
    _log("e2e")
    e2e = None
    if not args.no_e2e:
        e2e = bench_e2e(lib, gens, chains, steps, rank, world, dev, stream, max(1, args.steps // 2))
    _log("cpu baseline")
    cpu = None
    if rank == 0 and not args.no_cpu_baseline:  # after the timed region (also at N > 1)
        cpu = cpu_baseline_sample()

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": "evals/s", "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": step_ms,
                "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
                "dtype": "int32", "data": "synthetic",
                "config": {"workload": WORKLOAD.format(chains=chains, steps=steps), "n": N_JOBS,
                           "chains_per_gpu": chains,
                           "sa_steps": steps, "t0_samples": T0_SAMPLES, "instances": len(insts),
                           "parallelism": f"dp{world} (independent chains, NCCL min-allreduce)",
                           "l2": "state is on-chip; L2 flushed (256 MiB write) before every instance"},
                "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e,
                "gpu_launches": 4 * len(insts) * args.steps,
                "clocks": clk.summary(), "quality": gaps, **extra,
                "context": {"paper_gpu": "GeForce GT 560M", "paper_sa_evals_per_s_n1000": 2.22e5,
                            "paper_headline_speedup": "100x vs CPU [7] within 2% (P:7)"}}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def bench_dpso_multi_gpu(lib, cdist, dev, rank, world):
    """Config 4's swarm (CDD n=500, h=0.6, 8192 particles x 200 iterations) spread over all ranks,
    the swarm best global every iteration: exchanged by NCCL between launches, and fused into the
    kernels over peer memory (dpso_run_peer).  Device time, max over ranks; both give the same
    swarm (checked on the best)."""
    import torch
    import torch.distributed as dist

    import gen

    P, iters, seed = 8192 // world, 200, 0x5EED0004
    ins = lib.Instance.from_gen(gen.cdd_instance(500, 1, 0.6), device=dev.index)
    out = {"workload": f"config4: CDD n=500 h=0.6, DPSO {P * world} particles ({P} per GPU) x {iters} "
                       "iterations, swarm best global every iteration", "n_gpus": world}

    def timed(prep, fn):
        prep()
        torch.cuda.synchronize()
        dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        t = torch.tensor([e0.elapsed_time(e1)], device=dev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    run_nccl = lambda: cdist.dpso_run_distributed(ins, P, iters, seed=seed)  # noqa: E731
    timed(lambda: None, run_nccl)
    ms = timed(lambda: None, run_nccl)
    best_nccl = lib.best_get(ins)[0]
    out["nccl_exchange"] = {"ms": ms, "particle_evals_per_s": P * world * (iters + 1) / (ms / 1e3)}
    ok, why = 1, ""
    try:
        cdist.peer_exchange_open(ins)
    except Exception as e:  # IPC / peer access unavailable: every rank must skip the fused run
        ok, why = 0, str(e)[:200]
    flag = torch.tensor([ok], device=dev, dtype=torch.int32)
    dist.all_reduce(flag, op=dist.ReduceOp.MIN)
    if int(flag.item()) == 1:
        sw = lib.Dpso(ins, P, iters, seed=seed, particle_offset=rank * P)
        prep = lambda: lib.dpso_peer_reset(ins)  # noqa: E731
        timed(prep, lambda: sw.run_peer())
        ms = timed(prep, lambda: sw.run_peer())
        best = lib.best_get(ins)[0]
        out["p2p_exchange"] = {"ms": ms, "particle_evals_per_s": P * world * (iters + 1) / (ms / 1e3),
                               "same_best_as_nccl": best == best_nccl}
    else:
        out["p2p_exchange"] = {"unavailable": why or "another rank could not open the peer regions"}
    return out


def _timed(stream, fn, reps=1):
    import torch

    fn()  # warm-up (JIT of nothing, but allocations and first-launch costs)
    torch.cuda.synchronize()
    e1 = torch.cuda.Event(enable_timing=True)
    e2 = torch.cuda.Event(enable_timing=True)
    e1.record(stream)
    for _ in range(reps):
        fn()
    e2.record(stream)
    torch.cuda.synchronize()
    return e1.elapsed_time(e2) / reps / 1000.0


def bench_configs(lib, dev, stream):
    """Device throughput on the other BASELINE configs (one line each; CUDA-event timed)."""
    import numpy as np
    import torch

    import gen

    out = {}
    _log("  config 1: CDD n=10")
    # config 1: CDD n=10, h=0.4, seed 1 -- all 10! sequences + one 10k-step chain
    g1 = gen.cdd_instance(10, 1, 0.4)
    i1 = lib.Instance.from_gen(g1, device=dev.index)
    allp = torch.from_numpy(gen.all_perms(10)).to(dev)
    o1 = torch.empty(allp.shape[0], dtype=torch.int64, device=dev)
    t = _timed(stream, lambda: lib.cdd_eval_batch(i1, allp, o1), reps=5)
    t_sa = _timed(stream, lambda: lib.sa_run(i1, 1, 10000, seed=0x5EED0001))
    pen, _, _ = lib.best_get(i1)
    out["config1"] = {"exhaustive_evals_per_s": allp.shape[0] / t, "exhaustive_ms": 1000 * t,
                      "optimum": int(o1.min().item()), "sa_10k_chain_ms": 1000 * t_sa,
                      "sa_best": pen}
    _log("  config 2: CDD n=100, h in")
    # config 2: CDD n=100, h in {0.2..0.8} (instance 1): 1M random sequences + 4096 chains x 5000
    p2 = gen.random_perms_device(1 << 20, 100, 2, device=dev)
    o2 = torch.empty(p2.shape[0], dtype=torch.int64, device=dev)
    ev, sa = [], []
    for h in HS:
        ins = lib.Instance.from_gen(gen.cdd_instance(100, 1, h), device=dev.index)
        ev.append(p2.shape[0] / _timed(stream, lambda: lib.cdd_eval_batch(ins, p2, o2), reps=10))
        ws = lib.sa_run(ins, 4096, 5000, seed=0x5EED0002)["workspace"]
        dt = _timed(stream, lambda: lib.sa_run(ins, 4096, 5000, seed=0x5EED0002, workspace=ws))
        sa.append(4096 * 5001 / dt)
    out["config2"] = {"eval_batch_evals_per_s": sum(ev) / len(ev), "sa_evals_per_s": sum(sa) / len(sa),
                      "workload": "n=100, 4 h x instance 1; 2^20 random sequences; 4096 chains x 5000 steps"}
    _log("  config 3: UCDDCP n=200 unrestricted")
    # config 3: UCDDCP n=200 unrestricted, 16384 chains x 5000 steps
    i3 = lib.Instance.from_gen(gen.ucddcp_instance(200, 1), device=dev.index)
    ws = lib.sa_run(i3, 16384, 5000, problem="ucddcp", seed=0x5EED0003)["workspace"]
    dt = _timed(stream, lambda: lib.sa_run(i3, 16384, 5000, problem="ucddcp", seed=0x5EED0003,
                                           workspace=ws))
    out["config3"] = {"sa_evals_per_s": 16384 * 5001 / dt, "ms": 1000 * dt,
                      "workload": "UCDDCP n=200 (d = sum p), 16384 chains x 5000 steps"}
    _log("  config 4: CDD n=500, h=0.6: DPSO")
    # config 4: CDD n=500, h=0.6: DPSO 8192 particles vs SA at equal wall time (1 GPU)
    i4 = lib.Instance.from_gen(gen.cdd_instance(500, 1, 0.6), device=dev.index)
    iters = 200
    sw = lib.Dpso(i4, 8192, iters, seed=0x5EED0004)
    dt = _timed(stream, lambda: sw.run())
    dpso_best, _, _ = lib.best_get(i4)
    sa_rate_steps = 8192 * 200 / _timed(stream, lambda: lib.sa_run(i4, 8192, 200, seed=0x5EED0004))
    sa_steps = max(1, int(dt * sa_rate_steps / 8192))
    lib.sa_run(i4, 8192, sa_steps, seed=0x5EED0004)
    sa_best, _, _ = lib.best_get(i4)
    out["config4"] = {"dpso_particle_evals_per_s": 8192 * (iters + 1) / dt, "dpso_ms": 1000 * dt,
                      "dpso_best": dpso_best, "sa_steps_equal_time": sa_steps, "sa_best": sa_best,
                      "workload": "CDD n=500 h=0.6, DPSO 8192 particles x 200 iterations (w=c1=c2=0.5) vs "
                                  "8192 SA chains for the same wall time, 1 GPU"}
    _log("  synchronous SA (P:181-188)")
    # synchronous SA on the config-5 instance h=0.4: 65536 chains, M=50 x 100 levels
    # (5000 moves per chain, like SA_5000) vs asynchronous SA with the same moves
    i5 = lib.Instance.from_gen(gen.cdd_instance(N_JOBS, INSTANCE_SEED, 0.4), device=dev.index)
    ss = lib.SaSync(i5, 65536, 50, 100, seed=RUN_SEED, t0_samples=T0_SAMPLES, level_min=False)
    dt = _timed(stream, lambda: ss.run(), reps=1)
    sync_best, _, _ = lib.best_get(i5)
    lib.sa_run(i5, 65536, 5000, seed=RUN_SEED, t0_samples=T0_SAMPLES)
    async_best, _, _ = lib.best_get(i5)
    out["sync_sa"] = {"evals_per_s": 65536 * 5000 / dt, "ms": 1000 * dt, "best": sync_best,
                      "async_best_same_moves": async_best,
                      "workload": "synchronous SA, CDD n=1000 h=0.4, 65536 chains, M=50 moves x 100 "
                                  "temperature levels (mu per level)"}
    _log("  the headline SA from one V-shaped")
    # the headline SA from one V-shaped constructive sequence per chain instead of random ones
    # (sa_params.init; R13): quality only, same kernel and speed
    sys.path.insert(0, os.path.join(ROOT, "scripts"))
    from init_quality import v_shaped_candidates

    bk = {k: v["penalty"] for k, v in _best_known().items()}
    vq = {}
    for h in HS:
        g = gen.cdd_instance(N_JOBS, INSTANCE_SEED, h)
        ins = lib.Instance.from_gen(g, device=dev.index)
        cands = torch.from_numpy(v_shaped_candidates(g, np.linspace(0.2, 1.0, 33))).to(dev)
        s0 = cands[int(torch.argmin(lib.cdd_eval_batch(ins, cands)).item())].contiguous()
        lib.sa_run(ins, CHAINS, SA_STEPS, seed=RUN_SEED, t0_samples=T0_SAMPLES, init=s0)
        pen, _, _ = lib.best_get(ins)
        key = f"{h:.1f}"
        vq[key] = {"best": pen}
        if g.name() in bk:
            vq[key]["gap_pct"] = 100.0 * (pen - bk[g.name()]) / bk[g.name()]
    out["sa_from_v_shaped_start"] = {
        "quality": vq, "workload": "config 5 SA (65536 chains x 5000 steps) with every chain "
                                   "starting from one V-shaped constructive sequence (scripts/init_quality.py)"}
    return out


def _best_known():
    path = os.path.join(ROOT, "tests", "golden", "best_known.json")
    return json.load(open(path))["instances"] if os.path.exists(path) else {}


def bench_quality(lib, dev, stream):
    """SURVEY 8(d) quality outputs per BASELINE config, averaged over instances like Table II
    (40 instances per n): % gap of the best found to the oracle-verified best-known of
    tests/golden/best_known.json.  The paper's method: random initial sequences, mu = 0.88, T0 from
    5000 samples (configs 2, 3, 5: SA_5000; config 4: DPSO 8192 x 200 and SA for the same time)."""
    import torch

    import gen

    bk = _best_known()
    if not bk:
        return None

    def gap(g, pen):
        ref = bk.get(g.name(), {}).get("penalty")
        return None if ref is None else 100.0 * (pen - ref) / ref

    def summary(rows, **extra):
        gaps = [r for r in rows if r is not None]
        return {"mean_gap_pct": sum(gaps) / len(gaps) if gaps else None, "instances": len(gaps),
                "max_gap_pct": max(gaps) if gaps else None, **extra}

    out = {}
    t0 = time.time()
    _log("  config 2: CDD n=100, 10 instances")
    # config 2: CDD n=100, 10 instances x 4 h, 4096 chains x 5000 steps
    per_h = {f"{h:.1f}": [] for h in HS}
    for k in range(1, 11):
        for h in HS:
            g = gen.cdd_instance(100, k, h)
            ins = lib.Instance.from_gen(g, device=dev.index)
            lib.sa_run(ins, 4096, 5000, seed=0x5EED0002)
            per_h[f"{h:.1f}"].append(gap(g, lib.best_get(ins)[0]))
    out["config2"] = summary(sum(per_h.values(), []), per_h={k: summary(v)["mean_gap_pct"] for k, v in per_h.items()},
                             workload="CDD n=100, 10 instances x 4 h, SA 4096 chains x 5000 steps")
    _log("  config 3: UCDDCP n=200, 10 instances")
    # config 3: UCDDCP n=200, 10 instances, 16384 chains x 5000 steps
    rows = []
    for k in range(1, 11):
        g = gen.ucddcp_instance(200, k)
        ins = lib.Instance.from_gen(g, device=dev.index)
        lib.sa_run(ins, 16384, 5000, problem="ucddcp", seed=0x5EED0003)
        rows.append(gap(g, lib.best_get(ins)[0]))
    out["config3"] = summary(rows, workload="UCDDCP n=200 (d = sum p), 10 instances, SA 16384 chains x 5000 steps")
    _log("  config 4: CDD n=500 h=0.6, 10 instance")
    # config 4: CDD n=500 h=0.6, 10 instances: DPSO 8192 x 200 vs SA for the same wall time
    rd, rs = [], []
    for k in range(1, 11):
        g = gen.cdd_instance(500, k, 0.6)
        ins = lib.Instance.from_gen(g, device=dev.index)
        sw = lib.Dpso(ins, 8192, 200, seed=0x5EED0004)
        dt = _timed(stream, lambda: sw.run(), reps=1)
        rd.append(gap(g, lib.best_get(ins)[0]))
        rate = 8192 * 200 / _timed(stream, lambda: lib.sa_run(ins, 8192, 200, seed=0x5EED0004), reps=1)
        lib.sa_run(ins, 8192, max(1, int(dt * rate / 8192)), seed=0x5EED0004)
        rs.append(gap(g, lib.best_get(ins)[0]))
    out["config4"] = {"dpso": summary(rd), "sa_equal_time": summary(rs),
                      "workload": "CDD n=500 h=0.6, 10 instances; DPSO 8192 particles x 200 iterations "
                                  "(w=c1=c2=0.5) vs 8192 SA chains for the same wall time"}
    _log("  config 5: CDD n=1000, 10 instances")
    # config 5: CDD n=1000, 10 instances x 4 h, 65536 chains x 5000 steps (the headline workload)
    per_h = {f"{h:.1f}": [] for h in HS}
    for k in range(1, 11):
        for h in HS:
            g = gen.cdd_instance(N_JOBS, k, h)
            ins = lib.Instance.from_gen(g, device=dev.index)
            lib.sa_run(ins, CHAINS, SA_STEPS, seed=RUN_SEED, t0_samples=T0_SAMPLES)
            per_h[f"{h:.1f}"].append(gap(g, lib.best_get(ins)[0]))
    out["config5"] = summary(sum(per_h.values(), []), per_h={k: summary(v)["mean_gap_pct"] for k, v in per_h.items()},
                             workload=f"CDD n=1000, 10 instances x 4 h, SA {CHAINS} chains x {SA_STEPS} steps")
    _log("  the other neighbourhoods")
    # the other neighbourhoods on the same 40 instances (R11b insertion, R11c contiguous window of
    # Pert = 4 positions; swap) beside the paper's Pert-FY reading R11 above
    moves = {}
    for mv in ("window", "swap", "insert"):
        rows = []
        for k in range(1, 11):
            for h in HS:
                g = gen.cdd_instance(N_JOBS, k, h)
                ins = lib.Instance.from_gen(g, device=dev.index)
                lib.sa_run(ins, CHAINS, SA_STEPS, seed=RUN_SEED, t0_samples=T0_SAMPLES, move=mv)
                rows.append(gap(g, lib.best_get(ins)[0]))
        moves[mv] = summary(rows)
    out["config5"]["moves"] = moves
    out["seconds"] = time.time() - t0
    out["reference"] = ("% gap to tests/golden/best_known.json (best of long GPU searches, every penalty "
                        "re-evaluated by the oracle); the paper's Table II reports %Delta to [7]'s results "
                        "(P:282-300), not to optima")
    return out


def bench_eval(lib, g, dev, stream, peaks, batch=1 << 20, reps=20):
    """Batched evaluation kernel at n=1000 (HBM roofline), inputs 2 GiB >> L2."""
    import torch

    import gen

    ins = lib.Instance.from_gen(g, device=dev.index)
    pools = [gen.random_perms_device(batch, N_JOBS, 7 + i, device=dev) for i in range(2)]
    out = torch.empty(batch, dtype=torch.int64, device=dev)
    for i in range(3):
        lib.cdd_eval_batch(ins, pools[i % 2], out)
    torch.cuda.synchronize()
    e1 = torch.cuda.Event(enable_timing=True)
    e2 = torch.cuda.Event(enable_timing=True)
    e1.record(stream)
    for i in range(reps):
        lib.cdd_eval_batch(ins, pools[i % 2], out)
    e2.record(stream)
    torch.cuda.synchronize()
    ms = e1.elapsed_time(e2) / reps
    lib.cdd_check(ins)
    bytes_per = batch * (2 * N_JOBS + 8)
    gbs = bytes_per / (ms / 1000) / 1e9
    hbm = float(peaks.get("hbm_gbs", 6454.0))
    traffic = None
    tp = os.path.join(ROOT, "profiles", "eval_kernel_dram_bytes.json")
    if os.path.exists(tp):
        traffic = json.load(open(tp)).get("dram_bytes_per_launch")
    return {"workload": "cdd_eval_batch, CDD n=1000 h=0.4, 2^20 random sequences (2 GiB, alternating pools > L2)",
            "evals_per_s": batch / (ms / 1000), "ms_per_launch": ms,
            "roofline": {"bound": "hbm", "achieved": gbs, "peak": hbm, "unit": "GB/s",
                         "frac": gbs / hbm, "traffic": traffic, "bytes_per_launch": bytes_per,
                         "algorithmic_bytes_per_eval": 2 * N_JOBS + 8}}


def bench_e2e(lib, gens, chains, steps, rank, world, dev, stream, k):
    """Same metric through the public API with HOST buffers: instance upload, SA, best download."""
    import torch

    from paper_conf_ipps_awasthillw16_b200 import dist as cdist

    def step():
        h2d = d2h = 0
        for g in gens:
            ins = lib.Instance(g.P, g.alpha, g.beta, g.d, device=dev.index)  # host -> device
            h2d += 3 * 4 * g.n
            lib.sa_run(ins, chains, steps, seed=RUN_SEED, chain_offset=rank * chains)
            if world > 1:
                cdist.global_best_async(ins)  # no host sync between instances
            pen, perm, gid = lib.best_get(ins)  # device -> host
            d2h += 8 + 2 * g.n
            ins.destroy()
        return h2d, d2h

    step()
    torch.cuda.synchronize()
    if world > 1:
        torch.distributed.barrier()
    t = time.perf_counter()
    for _ in range(k):
        h2d, d2h = step()
    torch.cuda.synchronize()
    dt = time.perf_counter() - t
    if world > 1:
        tt = torch.tensor([dt], device=dev, dtype=torch.float64)
        torch.distributed.all_reduce(tt, op=torch.distributed.ReduceOp.MAX)
        dt = float(tt.item())
    evals = _evals_per_step(chains, steps, T0_SAMPLES, len(gens)) * k * world
    return {"value": evals / dt, "unit": "evals/s", "h2d_bytes_per_step": h2d,
            "d2h_bytes_per_step": d2h, "steps": k}


if __name__ == "__main__":
    main()
