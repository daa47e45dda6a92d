"""Layout experiment for the batched CDD evaluator at n > 512 (CDD_EVAL2_CFG = "warps:flat:kc_log2",
read per launch by libcdd): throughput over two > L2 pools and equality with the default layout.
python scripts/eval2_cfg.py [--n 1000] cfg1 cfg2 ..."""
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
    ap.add_argument("cfgs", nargs="+")
    ap.add_argument("--n", type=int, default=1000)
    ap.add_argument("--reps", type=int, default=7)
    a = ap.parse_args()
    dev = torch.device("cuda", 0)
    n = a.n
    inst = cdd.Instance.from_gen(gen.cdd_instance(n, 1, 0.4))
    ld = (n + 7) // 8 * 8
    rows = (1 << 31) // (2 * ld)
    pools = [gen.random_perms_device(rows, n, seed=s, ld=ld, device=dev) for s in (1, 2)]
    out = torch.empty(rows, dtype=torch.int64, device=dev)
    os.environ.pop("CDD_EVAL2_CFG", None)
    cdd.cdd_eval_batch(inst, pools[0], out)
    ref = out.clone()
    for cfg in ["default"] + a.cfgs:
        if cfg != "default":
            os.environ["CDD_EVAL2_CFG"] = cfg
        out.zero_()
        cdd.cdd_eval_batch(inst, pools[0], out)
        torch.cuda.synchronize()
        same = bool(torch.equal(out, ref))
        times = []
        for r in range(a.reps):
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            cdd.cdd_eval_batch(inst, pools[r & 1], out)
            e.record()
            torch.cuda.synchronize()
            times.append(s.elapsed_time(e))
        ms = sorted(times)[len(times) // 2]
        print(json.dumps({"cfg": cfg, "n": n, "same": same, "ms": round(ms, 4),
                          "evals_per_s": rows / (ms * 1e-3),
                          "GBps": rows * (2 * n + 8) / (ms * 1e-3) / 1e9}), flush=True)
    inst.destroy()


if __name__ == "__main__":
    main()
