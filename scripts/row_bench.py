"""One measurement per SURVEY §8 row that has a kernel of its own, each against the roofline that
bounds it (DESIGN.md §7 / §8): prints one JSON line per row.

  A7  cdd_eval_batch / ucddcp_eval_batch, n=1000: HBM (2n + 8 bytes per sequence)
  A8  T0 rule (5000 samples), n=1000: issue (6n integer ops per sampled evaluation)
  A9-A11 asynchronous SA, n=1000: issue (6n per evaluation; UCDDCP 9n)
  A13-A14 DPSO, n=500: issue (6n per particle evaluation)
  F1  cdd_schedule_batch, n=1000: HBM (2n read + 8n written + 16 bytes per sequence)
  F2  synchronous SA, n=1000: issue (6n per evaluation)

  S4  SA with the insertion / window moves (R11b / R11c), n=1000
  G   the generic ("wide") path: batched evaluation at n=1000 (warp per sequence) and n=4096 (CTA
      per sequence), asynchronous SA at n=1000

Peaks: MEASURED_PEAKS.json (HBM GB/s, SM max clock); integer peak = the best measured lane-op rate
of scripts/int_peak.cu (profiles/r2_int_peak.jsonl) x SMs x max clock.  Inputs larger than L2 for
the HBM rows (two alternating pools).
python scripts/row_bench.py [ROW ...]   (default: every row; e.g. `G S4`)"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_awasthillw16_b200 as cdd  # noqa: E402


def timed(fn, reps=5):
    fn()
    torch.cuda.synchronize()
    ts = []
    for r in range(reps):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        fn(r)
        e.record()
        torch.cuda.synchronize()
        ts.append(s.elapsed_time(e) / 1000.0)
    return sorted(ts)[len(ts) // 2]


def main():
    sel = set(sys.argv[1:])

    def want(row):
        return not sel or row in sel

    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {}
    hbm = float(peaks.get("hbm_gbs", 6454.0))
    sm_mhz = float(peaks.get("sm_max_mhz", 1965.0))
    nsm = torch.cuda.get_device_properties(0).multi_processor_count
    ip = [json.loads(x) for x in open(os.path.join(ROOT, "profiles", "r2_int_peak.jsonl")) if x.startswith("{")]
    lane_ops = max(r["lane_ops_per_clk_per_sm"] for r in ip)
    alu = lane_ops * nsm * sm_mhz * 1e6 / 1e12  # T int-op/s (measured)

    def out(row, what, value, unit, achieved, peak, punit, note=""):
        # HBM rows: algorithmic bytes against the measured copy bandwidth (a fraction).  Integer
        # rows: the SURVEY 8(d) algorithmic op count against the int32 lane-op peak -- a ratio,
        # not a fraction, since the byte-SIMD kernels do up to four such ops per lane-op (the
        # issue-based fraction of the headline kernel is in bench.py's roofline)
        key = "frac" if punit == "GB/s" else "algorithmic_ratio"
        print(json.dumps({"row": row, "what": what, "value": value, "unit": unit,
                          "roofline": {"achieved": achieved, "peak": peak, "unit": punit,
                                       key: achieved / peak}, "note": note}), flush=True)

    n = 1000
    rows = 1 << 20
    pools = [gen.random_perms_device(rows, n, seed=s, ld=n) for s in (1, 2)]
    o = torch.empty(rows, dtype=torch.int64, device="cuda")
    ic = cdd.Instance.from_gen(gen.cdd_instance(n, 1, 0.4))
    iu = cdd.Instance.from_gen(gen.ucddcp_instance(n, 1))
    for name, ins, fn in ((("cdd_eval_batch", ic, cdd.cdd_eval_batch), ("ucddcp_eval_batch", iu, cdd.ucddcp_eval_batch))
                          if want("A7") else ()):
        dt = timed(lambda r=0: fn(ins, pools[r & 1], o), reps=9)
        gbs = rows * (2 * n + 8) / dt / 1e9
        out("A7" if name.startswith("cdd") else "A6/A7", f"{name} n={n}, 2^20 sequences", rows / dt,
            "evals/s", gbs, hbm, "GB/s")
    cdd.cdd_check(ic)
    cdd.cdd_check(iu)

    # F1 schedules: C int64 [B, n] written, sequences read
    B = 1 << 17
    sp = pools[0][:B]
    if want("F1"):
        dt = timed(lambda r=0: cdd.cdd_schedule_batch(ic, sp), reps=5)
        out("F1", f"cdd_schedule_batch n={n}, 2^17 sequences", B / dt, "schedules/s",
            B * (2 * n + 8 * n + 16) / dt / 1e9, hbm, "GB/s", "C int64 [B, n] written + start + penalty")
        dt = timed(lambda r=0: cdd.cdd_schedule_batch(iu, sp, "ucddcp"), reps=5)
        out("F1", f"ucddcp schedule_batch n={n}, 2^17 sequences", B / dt, "schedules/s",
            B * (2 * n + 12 * n + 16) / dt / 1e9, hbm, "GB/s",
            "C int64 + X int32 [B, n] written + start + penalty")

    # A8 T0
    T0 = 5000
    if want("A8"):
        dt = timed(lambda r=0: cdd.sa_t0(ic, seed=r, samples=T0), reps=9)
        out("A8", f"T0 rule, {T0} samples, n={n}", T0 / dt, "samples/s", 6 * n * T0 / dt / 1e12, alu,
            "Tint-op/s", "one launch pair: small grid (5000 warps), latency-bound")

    # A9-A11 SA (CDD and UCDDCP)
    for prob, ins, ops in (("cdd", ic, 6), ("ucddcp", iu, 9)) if want("A9") else ():
        C, S = 65536, 1000
        t0 = cdd.sa_t0(ins, problem=prob, seed=1, samples=T0)
        ws = cdd.sa_run(ins, C, S, problem=prob, seed=1, T0_dev=t0)["workspace"]
        dt = timed(lambda r=0: cdd.sa_run(ins, C, S, problem=prob, seed=1, T0_dev=t0, workspace=ws), reps=3)
        ev = C * (S + 1)
        out("A9-A11", f"SA {prob} n={n}, {C} chains x {S} steps", ev / dt, "evals/s",
            ops * n * ev / dt / 1e12, alu, "Tint-op/s", f"{ops}n algorithmic int ops per evaluation")

    # the headline SA with the byte-row layout (CDD_SA_NO_NIB=1: no 4-bit weights, no sub-block
    # summaries) for comparison with the small-weight layout the row above uses
    if want("A9"):
        C, S = 65536, 1000
        os.environ["CDD_SA_NO_NIB"] = "1"
        try:
            t0 = cdd.sa_t0(ic, seed=1, samples=T0)
            ws = cdd.sa_run(ic, C, S, seed=1, T0_dev=t0)["workspace"]
            dt = timed(lambda r=0: cdd.sa_run(ic, C, S, seed=1, T0_dev=t0, workspace=ws), reps=3)
        finally:
            del os.environ["CDD_SA_NO_NIB"]
        ev = C * (S + 1)
        out("A9-A11", f"SA cdd n={n} byte-row layout (CDD_SA_NO_NIB=1), {C} chains x {S} steps", ev / dt,
            "evals/s", 6 * n * ev / dt / 1e12, alu, "Tint-op/s", "6n algorithmic int ops per evaluation")

    # F2 synchronous SA
    C, M, L = 65536, 50, 20
    if want("F2"):
        ss = cdd.SaSync(ic, C, M, L, seed=3, t0_samples=T0, level_min=False)
        dt = timed(lambda r=0: ss.run(), reps=3)
        ev = C * M * L
        out("F2", f"synchronous SA n={n}, {C} chains, M={M} x {L} levels", ev / dt, "evals/s",
            6 * n * ev / dt / 1e12, alu, "Tint-op/s")

    # A13-A14 DPSO
    for n2 in (100, 500, 1000) if want("A13") else ():
        i5 = cdd.Instance.from_gen(gen.cdd_instance(n2, 1, 0.6))
        P, it = 8192, 200
        sw = cdd.Dpso(i5, P, it, seed=4)
        dt = timed(lambda r=0: sw.run(), reps=3)
        ev = P * (it + 1)
        out("A13-A14", f"DPSO n={n2}, {P} particles x {it} iterations", ev / dt, "particle-evals/s",
            6 * n2 * ev / dt / 1e12, alu, "Tint-op/s", "per iteration: F1-F3 + evaluation + swarm best")

    # S4: the other moves on the headline instance
    for mv in ("insert", "window", "swap") if want("S4") else ():
        C, S = 65536, 1000
        t0 = cdd.sa_t0(ic, seed=1, samples=T0)
        ws = cdd.sa_run(ic, C, S, seed=1, T0_dev=t0, move=mv)["workspace"]
        dt = timed(lambda r=0: cdd.sa_run(ic, C, S, seed=1, T0_dev=t0, workspace=ws, move=mv), reps=3)
        ev = C * (S + 1)
        out("S4", f"SA cdd n={n} move={mv}, {C} chains x {S} steps", ev / dt, "evals/s",
            6 * n * ev / dt / 1e12, alu, "Tint-op/s")

    # G: generic path (values outside the packed ranges)
    import numpy as np

    rng = np.random.default_rng(5)
    for nw, batch in ((1000, 1 << 18), (4096, 1 << 14)) if want("G") else ():
        P = rng.integers(1, 1001, nw).astype(np.int32)
        a = rng.integers(1, 10001, nw).astype(np.int32)
        b = rng.integers(1, 10001, nw).astype(np.int32)
        iw = cdd.Instance(P, a, b, int(0.4 * int(P.sum())))
        assert iw.wide
        pw = [gen.random_perms_device(batch, nw, seed=s, ld=nw) for s in (3, 4)]
        ow = torch.empty(batch, dtype=torch.int64, device="cuda")
        dt = timed(lambda r=0: cdd.cdd_eval_batch(iw, pw[r & 1], ow), reps=5)
        out("G", f"generic cdd_eval_batch n={nw} (p<=1000, alpha,beta<=1e4), {batch} sequences", batch / dt,
            "evals/s", batch * (2 * nw + 8) / dt / 1e9, hbm, "GB/s",
            "int64 arithmetic, int4 record gathers from L1/L2 (one pass)")
        if nw == 1000:
            C, S = 16384, 200
            ws = cdd.sa_run(iw, C, S, seed=1, T0=1e9)["workspace"]
            dt = timed(lambda r=0: cdd.sa_run(iw, C, S, seed=1, T0=1e9, workspace=ws), reps=3)
            ev = C * (S + 1)
            out("G", f"generic SA n={nw}, {C} chains x {S} steps", ev / dt, "evals/s",
                6 * nw * ev / dt / 1e12, alu, "Tint-op/s", "one warp per chain, ids in L2")


if __name__ == "__main__":
    main()
