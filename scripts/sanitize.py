"""Small runs of every kernel family for compute-sanitizer (memcheck / racecheck / synccheck):
python scripts/sanitize.py  (under `compute-sanitizer --tool X python scripts/sanitize.py`)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_awasthillw16_b200 as cdd  # noqa: E402

for n in (7, 50, 100, 200, 500, 777, 1000):
    ins = cdd.Instance.from_gen(gen.cdd_instance(n, 1, 0.4))
    perms = gen.random_perms_device(700, n, 3, ld=(n + 7) // 8 * 8)
    cdd.cdd_eval_batch(ins, perms)
    cdd.cdd_schedule_batch(ins, perms[:50])
    cdd.sa_run(ins, 300, 20, seed=1, t0_samples=100)
    cdd.sa_run(ins, 40, 20, seed=1, t0_samples=100, lanes=32, init=perms[0])
    if n >= 2:
        cdd.dpso_run(ins, 64, 5, seed=2)
    cdd.SaSync(ins, 64, 5, 3, seed=3, t0_samples=100).run()
    cdd.SaSync(ins, 1024, 4, 3, seed=3, t0_samples=100).run()  # group kernel + level images
    cdd.cdd_check(ins)
    u = cdd.Instance.from_gen(gen.ucddcp_instance(n, 1))
    cdd.ucddcp_eval_batch(u, perms)
    cdd.cdd_schedule_batch(u, perms[:50], "ucddcp")
    cdd.sa_run(u, 300, 20, problem="ucddcp", seed=1, t0_samples=100)
    if n >= 2:
        cdd.dpso_run(u, 64, 5, problem="ucddcp", seed=2)
    cdd.cdd_check(u)
# the small-weight SA layout (csrc/sa_nib.cuh: 4-bit weights, sub-block summaries, lane-pair
# recomputation) at G = 8, E = 128: every move of <= 4 positions, synchronous levels
for n in (600, 1000):
    ins = cdd.Instance.from_gen(gen.cdd_instance(n, 3, 0.6))
    assert ins.query()["small_weights"]
    for mv, pert in (("pert_fy", 4), ("swap", 2), ("window", 4), ("pert_fy", 3)):
        cdd.sa_run(ins, 64, 12, seed=5, t0_samples=100, lanes=8, move=mv, pert=pert)
    cdd.sa_run(ins, 64, 12, seed=5, t0_samples=100, lanes=8, trace=True)
    cdd.SaSync(ins, 64, 6, 3, seed=3, t0_samples=100, lanes=8).run()
    cdd.cdd_check(ins)
# balanced SA schedule (chains split between warps, state handed over): more chains than slots
ins = cdd.Instance.from_gen(gen.cdd_instance(120, 2, 0.4))
cdd.sa_run(ins, 15000, 9, seed=4, T0=900.0, lanes=8)
cdd.cdd_check(ins)
# fused exchange entry points on one rank (world 1), T0 on the group layout via sa_t0
ins = cdd.Instance.from_gen(gen.cdd_instance(300, 2, 0.4))
cdd.sa_t0(ins, samples=700)
h = cdd.dpso_peer_create(ins, 1, 0)
cdd.dpso_peer_open(ins, [h])
cdd.dpso_peer_reset(ins)
cdd.Dpso(ins, 64, 4, seed=2).run_peer()
cdd.dpso_peer_reset(ins)
cdd.SaSync(ins, 1024, 3, 2, seed=3, t0_samples=100).run_peer()
cdd.dpso_peer_destroy(ins)
cdd.cdd_check(ins)
# the insertion and window moves (R11b, R11c)
ins = cdd.Instance.from_gen(gen.cdd_instance(1000, 3, 0.4))
for mv in ("insert", "window"):
    cdd.sa_run(ins, 256, 30, seed=5, t0_samples=100, move=mv)
    cdd.sa_run(ins, 40, 30, seed=5, t0_samples=100, move=mv, lanes=32)
cdd.cdd_check(ins)
# the generic path (values outside the packed ranges; n up to 32767)
import numpy as np  # noqa: E402

rng = np.random.default_rng(7)
for nw in (300, 1500, 5000):
    P = rng.integers(1, 1001, nw).astype(np.int32)
    a = rng.integers(1, 10001, nw).astype(np.int32)
    b = rng.integers(1, 10001, nw).astype(np.int32)
    M = (P - rng.integers(0, P)).astype(np.int32)
    g = rng.integers(1, 10001, nw).astype(np.int32)
    for d in (int(0.4 * int(P.sum())), int(P.sum()) + 3):
        iw = cdd.Instance(P, a, b, d, M, g)
        pw = gen.random_perms_device(40, nw, 9, ld=nw)
        cdd.cdd_eval_batch(iw, pw)
        cdd.cdd_schedule_batch(iw, pw[:8])
        if d > int(P.sum()):
            cdd.ucddcp_eval_batch(iw, pw)
            cdd.cdd_schedule_batch(iw, pw[:8], "ucddcp")
        if nw <= 1500:
            cdd.sa_run(iw, 64, 10, seed=6, t0_samples=50, move="insert" if nw == 300 else "pert_fy")
        cdd.cdd_check(iw)
torch.cuda.synchronize()
print("sanitize run ok")
