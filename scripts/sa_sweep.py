"""SA throughput sweep over n (and problem) on one GPU: sequence evaluations/s of sa_run with an
explicit T0 (no T0 pass), timed with CUDA events.  Used for layout choices (lanes per chain).
python scripts/sa_sweep.py [--problem cdd|ucddcp] [--chains C] [--steps S] n1 n2 ..."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_awasthillw16_b200 as cdd  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("ns", type=int, nargs="+")
    ap.add_argument("--problem", default="cdd")
    ap.add_argument("--chains", type=int, default=65536)
    ap.add_argument("--steps", type=int, default=2000)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--lanes", type=int, default=0, help="threads per chain (0 automatic)")
    a = ap.parse_args()
    for n in a.ns:
        g = gen.ucddcp_instance(n, 1) if a.problem == "ucddcp" else gen.cdd_instance(n, 1, 0.4)
        inst = cdd.Instance.from_gen(g)
        ws = None
        cdd.sa_run(inst, 1024, 10, problem=a.problem, T0=5.0)  # warm-up / module load
        times = []
        for r in range(a.reps):
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            s.record()
            res = cdd.sa_run(inst, a.chains, a.steps, problem=a.problem, T0=50.0, seed=r,
                             workspace=ws, lanes=a.lanes)
            e.record()
            torch.cuda.synchronize()
            ws = res["workspace"]
            times.append(s.elapsed_time(e))
        ms = min(times)
        print(json.dumps({"n": n, "problem": a.problem, "lanes": a.lanes, "chains": a.chains,
                          "steps": a.steps,
                          "ms": round(ms, 3),
                          "evals_per_s": a.chains * a.steps / (ms * 1e-3),
                          "best": cdd.best_get(inst)[0]}))
        inst.destroy()


if __name__ == "__main__":
    main()
