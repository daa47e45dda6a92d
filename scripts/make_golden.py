"""Writes tests/golden/config1.json using ONLY the oracle (no CUDA path involved).

Config 1 of BASELINE.json: CDD n=10, h=0.4, generated instance seed 1 -- the exhaustive 10!
optimum (BASELINE.json north_star: "all n! permutations" brute force).
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import gen  # noqa: E402
import oracle  # noqa: E402


def main():
    inst = gen.cdd_instance(10, 1, 0.4)
    pr = oracle.Problem.from_instance(inst)
    perms = gen.all_perms(10)
    Z = oracle.eval_batch_threaded(pr, perms)
    zmin = int(Z.min())
    arg = int(np.argmin(Z))
    out = {
        "source": "scripts/make_golden.py (oracle only): exhaustive evaluation of all 10! sequences",
        "instance": {"n": 10, "seed": 1, "h": 0.4, "P": inst.P.tolist(), "alpha": inst.alpha.tolist(),
                     "beta": inst.beta.tolist(), "d": inst.d},
        "optimum": zmin,
        "n_optimal_sequences": int((Z == zmin).sum()),
        "first_optimal_sequence": perms[arg, :10].tolist(),
        "z_sum_over_all": int(Z.sum()),
        "z_max": int(Z.max()),
    }
    path = os.path.join(ROOT, "tests", "golden", "config1.json")
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
