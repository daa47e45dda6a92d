"""DPSO throughput (particle evaluations/s) on one GPU: python scripts/dpso_time.py [n ...]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_awasthillw16_b200 as cdd  # noqa: E402

for n in [int(x) for x in sys.argv[1:]] or [500]:
    inst = cdd.Instance.from_gen(gen.cdd_instance(n, 1, 0.6))
    P, iters = 8192, 200
    sw = cdd.Dpso(inst, P, iters, seed=4)
    sw.run()
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    sw.run()
    e.record()
    torch.cuda.synchronize()
    ms = s.elapsed_time(e)
    print(json.dumps({"n": n, "particles": P, "iters": iters, "ms": round(ms, 3),
                      "particle_evals_per_s": P * (iters + 1) / (ms * 1e-3),
                      "best": cdd.best_get(inst)[0]}))
