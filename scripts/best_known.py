"""Writes tests/golden/best_known_n1000.json using ONLY the oracle (no CUDA path involved).

"Best-known" penalties for the four bench instances (CDD n=1000, instance seed 1, h in
{0.2,0.4,0.6,0.8}): the minimum over long oracle SA runs (Alg. 1), every result re-evaluated with
the oracle's walk.  The OR-library best-knowns of [7] are not available offline.
Usage: python scripts/best_known.py [steps] [chains]
"""
import json
import os
import sys
import threading
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import gen  # noqa: E402
import oracle  # noqa: E402


def main():
    steps = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
    chains = int(sys.argv[2]) if len(sys.argv) > 2 else os.cpu_count() or 8
    out = {"source": "scripts/best_known.py (oracle SA only)", "steps": steps, "chains": chains,
           "runs": {}, "best_known": {}}
    for h in (0.2, 0.4, 0.6, 0.8):
        inst = gen.cdd_instance(1000, 1, h)
        pr = oracle.Problem.from_instance(inst)
        T0 = oracle.t0(pr, oracle.CDD, 0xB357, 5000)
        results = {}
        t = time.time()
        for mu in (0.88, 0.99999):
            res = [None] * chains

            def work(c, mu=mu, res=res):
                p = oracle.sa_params(steps=steps, mu=mu, seed=0xB357 + int(mu * 1e5))
                r = oracle.sa_chain(pr, p, T0, c)
                res[c] = (r["E_best"], r["best"])

            ts = [threading.Thread(target=work, args=(c,)) for c in range(chains)]
            [x.start() for x in ts]
            [x.join() for x in ts]
            eb, J = min(res, key=lambda x: x[0])
            assert oracle.cdd_eval(pr, J) == eb
            results[str(mu)] = eb
        key = f"{h:.1f}"
        out["runs"][key] = results
        out["best_known"][key] = min(results.values())
        print(key, results, f"{time.time() - t:.0f}s", flush=True)
    with open(os.path.join(ROOT, "tests", "golden", "best_known_n1000.json"), "w") as f:
        json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
