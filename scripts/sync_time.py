"""Synchronous-SA cost decomposition: same total moves per chain split into different (M, levels),
and chain counts around the resident-slot count.  python scripts/sync_time.py"""
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
    ts = []
    for _ in range(reps):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        fn()
        e.record()
        torch.cuda.synchronize()
        ts.append(s.elapsed_time(e) * 1e-3)
    return sorted(ts)[len(ts) // 2]


def main():
    n = 1000
    ic = cdd.Instance.from_gen(gen.cdd_instance(n, 1, 0.4))
    for C, M, L in [(65536, 50, 20), (65536, 100, 10), (65536, 250, 4), (65536, 1000, 1),
                    (65536, 50, 1), (65536, 50, 2), (9472, 50, 20), (9472, 1000, 1)]:
        ss = cdd.SaSync(ic, C, M, L, seed=3, T0=1000.0, level_min=False)
        dt = timed(lambda: ss.run())
        print(json.dumps({"chains": C, "M": M, "levels": L, "ms": dt * 1e3,
                          "evals_per_s": C * M * L / dt}))
    for C, S in [(65536, 1000), (65536, 50), (9472, 1000)]:
        dt = timed(lambda: cdd.sa_run(ic, C, S, seed=3, T0=1000.0))
        print(json.dumps({"async_chains": C, "steps": S, "ms": dt * 1e3, "evals_per_s": C * S / dt}))


if __name__ == "__main__":
    main()
