"""Batched-evaluation throughput sweep over n on one GPU: cdd_eval_batch / ucddcp_eval_batch over
two pools of random sequences (each larger than L2, alternated), timed with CUDA events.
python scripts/eval_sweep.py [--problem cdd|ucddcp] [--rows R] [--reps K] n1 n2 ..."""
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
    ap.add_argument("--rows", type=int, default=1 << 20)
    ap.add_argument("--reps", type=int, default=5)
    a = ap.parse_args()
    fn = cdd.ucddcp_eval_batch if a.problem == "ucddcp" else cdd.cdd_eval_batch
    dev = torch.device("cuda", 0)
    for n in a.ns:
        g = gen.ucddcp_instance(n, 1) if a.problem == "ucddcp" else gen.cdd_instance(n, 1, 0.4)
        inst = cdd.Instance.from_gen(g)
        ld = (n + 15) // 16 * 16
        rows = max(1024, min(a.rows, (1 << 31) // (2 * ld)))
        pools = [gen.random_perms_device(rows, n, seed=s, ld=ld, device=dev) for s in (1, 2)]
        out = torch.empty(rows, dtype=torch.int64, device=dev)
        fn(inst, pools[0], out)
        torch.cuda.synchronize()
        times = []
        for r in range(a.reps):
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            fn(inst, pools[r & 1], out)
            e.record()
            torch.cuda.synchronize()
            times.append(s.elapsed_time(e))
        ms = sorted(times)[len(times) // 2]
        print(json.dumps({"n": n, "problem": a.problem, "rows": rows, "ld": ld, "ms": round(ms, 4),
                          "evals_per_s": rows / (ms * 1e-3),
                          "GBps": rows * (2 * ld + 8) / (ms * 1e-3) / 1e9}))
        inst.destroy()


if __name__ == "__main__":
    main()
