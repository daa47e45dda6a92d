"""DPSO time per iteration against the swarm size (n = 500): the per-iteration floor (grid barrier,
swarm-best publish) shows at small swarms.  python scripts/dpso_floor.py"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_awasthillw16_b200 as cdd  # noqa: E402

inst = cdd.Instance.from_gen(gen.cdd_instance(int(sys.argv[1]) if len(sys.argv) > 1 else 500, 1, 0.6))
for P in (148, 592, 2368, 4736, 8192, 9472):
    for c in ((0.5, 0.5, 0.5), (0.0, 0.0, 0.0), (1.0, 1.0, 1.0)):
        iters = 200
        sw = cdd.Dpso(inst, P, iters, seed=4, w=c[0], c1=c[1], c2=c[2])
        sw.run()
        torch.cuda.synchronize()
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        sw.run()
        e.record()
        torch.cuda.synchronize()
        ms = s.elapsed_time(e)
        print(json.dumps({"particles": P, "w_c1_c2": c, "us_per_iter": round(1000 * ms / iters, 2),
                          "particle_evals_per_s": P * (iters + 1) / (ms * 1e-3)}), flush=True)
