"""F1 schedule throughput (cdd_schedule_batch) at n=1000, 2^17 sequences, CDD and UCDDCP:
python scripts/sched_time.py"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_awasthillw16_b200 as cdd  # noqa: E402

peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
    os.path.join(ROOT, "MEASURED_PEAKS.json")) else {}
hbm = float(peaks.get("hbm_gbs", 6454.0))
n, B = 1000, 1 << 17
pools = [gen.random_perms_device(B, n, seed=s, ld=n) for s in (1, 2)]
for prob, g in (("cdd", gen.cdd_instance(n, 1, 0.4)), ("ucddcp", gen.ucddcp_instance(n, 1))):
    ins = cdd.Instance.from_gen(g)
    cdd.cdd_schedule_batch(ins, pools[0], prob)
    torch.cuda.synchronize()
    ts = []
    for r in range(6):
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        cdd.cdd_schedule_batch(ins, pools[r & 1], prob)
        e.record()
        torch.cuda.synchronize()
        ts.append(s.elapsed_time(e) / 1e3)
    dt = sorted(ts)[len(ts) // 2]
    bytes_ = B * (2 * n + 8 * n + 16 + (4 * n if prob == "ucddcp" else 0))
    print(json.dumps({"problem": prob, "n": n, "batch": B, "schedules_per_s": B / dt,
                      "gbs": bytes_ / dt / 1e9, "frac_hbm": bytes_ / dt / 1e9 / hbm}), flush=True)
