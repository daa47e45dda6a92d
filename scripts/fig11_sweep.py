"""F4: the paper's Fig. 11 study re-done on B200 -- SA runtime on the UCDDCP as a
function of the number of chains (the paper's threads = population) and iterations
(generations), plus the layout axis B200 adds (threads per chain).  Writes one JSON object per
line; `--md` prints a markdown table as well.

python scripts/fig11_sweep.py [--n 200] [--md]"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_awasthillw16_b200 as cdd  # noqa: E402


def timed(fn, reps=3):
    fn()
    torch.cuda.synchronize()
    best = None
    for _ in range(reps):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        fn()
        e.record()
        torch.cuda.synchronize()
        t = s.elapsed_time(e)
        best = t if best is None else min(best, t)
    return best


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=200)
    ap.add_argument("--problem", default="ucddcp")
    ap.add_argument("--md", action="store_true")
    a = ap.parse_args()
    g = gen.ucddcp_instance(a.n, 1) if a.problem == "ucddcp" else gen.cdd_instance(a.n, 1, 0.4)
    inst = cdd.Instance.from_gen(g)
    T0 = cdd.sa_t0(inst, a.problem, seed=1, samples=5000)
    rows = []
    for chains in (768, 4096, 16384, 65536, 262144):
        for steps in (1000, 5000):
            for lanes in (0, 32, 16, 8, 4):
                if lanes == 4 and a.n > 256:
                    continue
                ms = timed(lambda: cdd.sa_run(inst, chains, steps, problem=a.problem, seed=1,
                                              T0_dev=T0, lanes=lanes))
                G, E = cdd.sa_layout(inst, chains, a.problem, lanes)
                best = cdd.best_get(inst)[0]
                r = {"n": a.n, "problem": a.problem, "chains": chains, "steps": steps,
                     "lanes_arg": lanes, "lanes": G, "positions_per_lane": E, "ms": round(ms, 3),
                     "evals_per_s": chains * (steps + 1) / (ms * 1e-3), "best": best}
                rows.append(r)
                print(json.dumps(r), flush=True)
    if a.md:
        print(f"\n| chains | steps | auto (lanes) | 32 | 16 | 8 | 4 | best (auto) |")
        print("|---|---|---|---|---|---|---|---|")
        for chains in (768, 4096, 16384, 65536, 262144):
            for steps in (1000, 5000):
                rs = {r["lanes_arg"]: r for r in rows if r["chains"] == chains and r["steps"] == steps}
                cell = lambda k: f"{rs[k]['ms']:.2f} ms" if k in rs else "-"  # noqa: E731
                print(f"| {chains} | {steps} | {cell(0)} ({rs[0]['lanes']}) | {cell(32)} | {cell(16)} | "
                      f"{cell(8)} | {cell(4)} | {rs[0]['best']} |")


if __name__ == "__main__":
    main()
