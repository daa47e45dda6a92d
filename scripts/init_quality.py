"""Quality of asynchronous SA at n=1000 (bench config 5) by initial sequences (sa_params.init):
R13's random sequence per chain vs one V-shaped constructive sequence for every chain.

The paper does not say where its initial sequences come from ("the initial job sequences are
copied to the GPU"; "the same or different for all chains").  This script measures
how much that choice matters.  The V-shaped sequence is a user-side construction, not part of the
library: jobs ranked by (beta - alpha) / p fill the early side while their processing times fit
before a cap (the due date, and at most a fraction f of the total), the early side is ordered by
p/alpha descending and the tardy side by p/beta ascending (the V-shape of optimal CDD schedules,
P:77-92); the best f over a small grid is taken with the batched evaluator.

python scripts/init_quality.py [--chains 65536] [--steps 5000]"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_awasthillw16_b200 as cdd  # noqa: E402


def v_shaped_candidates(g, fracs):
    P, a, b = g.P.astype(float), g.alpha.astype(float), g.beta.astype(float)
    rank = np.argsort(-(b - a) / P, kind="stable")
    out = []
    for f in fracs:
        cap = min(float(g.d), f * P.sum())
        early, tardy, used = [], [], 0.0
        for j in rank:
            if used + P[j] <= cap:
                early.append(j)
                used += P[j]
            else:
                tardy.append(j)
        early.sort(key=lambda j: -P[j] / a[j] if a[j] > 0 else -np.inf)
        tardy.sort(key=lambda j: P[j] / b[j] if b[j] > 0 else np.inf)
        out.append(np.array(early + tardy, dtype=np.int16))
    return np.stack(out)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--chains", type=int, default=65536)
    ap.add_argument("--steps", type=int, default=5000)
    a = ap.parse_args()
    bk = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                     "tests", "golden", "best_known_n1000.json")))["best_known"]
    for h in (0.2, 0.4, 0.6, 0.8):
        g = gen.cdd_instance(1000, 1, h)
        ins = cdd.Instance.from_gen(g)
        cands = torch.from_numpy(v_shaped_candidates(g, np.linspace(0.2, 1.0, 33))).cuda()
        z = cdd.cdd_eval_batch(ins, cands)
        s0 = cands[int(torch.argmin(z).item())].contiguous()
        ref = bk[f"{h:.1f}"]
        row = {"h": h, "best_known": ref, "v_shape_start": int(z.min().item())}
        for name, init in (("random_starts", None), ("v_shape_start_sa", s0)):
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            cdd.sa_run(ins, a.chains, a.steps, seed=0x5EED0005, init=init)
            e.record()
            torch.cuda.synchronize()
            pen = cdd.best_get(ins)[0]
            row[name] = {"best": pen, "gap_pct": round(100.0 * (pen - ref) / ref, 3),
                         "ms": round(s.elapsed_time(e), 2)}
        print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
