"""OR-library CDD benchmark files (Biskup & Feldmann, `sch10.txt` ... `sch1000.txt`; SURVEY §8(f) F3,
P:261) and the run-and-compare loop of Tables II/IV.

File format (OR-library `schinfo`): the number of problems K, then for each problem the number of
jobs n followed by n lines `p a b` (processing time, earliness and tardiness penalty); all
integers, whitespace separated.  The due date of problem k at restrictive factor h is
d = floor(h * sum p) (h in {0.2, 0.4, 0.6, 0.8}).  This loader is host-side input handling;
the search itself runs in libcdd (sa_run / dpso_run).

UCDDCP instances ([8]) are read from the same layout with five columns per job,
`P M a b gamma` -- the column order is an assumption (the published files were not available
offline), so `read_ucddcp` takes an explicit `columns` argument.

CLI: python -m paper_conf_ipps_awasthillw16_b200.orlib FILE --k 1 --h 0.4 [--chains C --steps S
     --best-known Z]  ->  one JSON line with the best penalty and its % deviation (Table II's
     Delta = 100 (Z - Z_bk) / Z_bk)."""
from __future__ import annotations

import argparse
import dataclasses
import json
import math
import sys

import numpy as np


@dataclasses.dataclass
class OrInstance:
    """One benchmark problem: job data by job id (and the due date once h is chosen)."""
    n: int
    P: np.ndarray
    alpha: np.ndarray
    beta: np.ndarray
    M: np.ndarray | None = None
    gamma: np.ndarray | None = None
    d: int | None = None
    k: int = 1          # 1-based problem number in its file
    h: float | None = None

    def with_h(self, h: float) -> "OrInstance":
        """Restrictive factor h: d = floor(h * sum p) in exact integer arithmetic."""
        num = round(h * 10)
        if abs(num - 10 * h) > 1e-9:
            d = math.floor(h * int(self.P.sum()))
        else:
            d = (num * int(self.P.sum())) // 10
        return dataclasses.replace(self, d=d, h=h)


def _ints(text: str) -> list[int]:
    try:
        return [int(t) for t in text.split()]
    except ValueError as e:
        raise ValueError(f"OR-library file: non-integer token ({e})") from None


def parse_sch(text: str, columns: int = 3) -> list[OrInstance]:
    """All problems of an OR-library sch file (columns = 3: p a b)."""
    v = _ints(text)
    if not v:
        raise ValueError("OR-library file: empty")
    K, pos, out = v[0], 1, []
    if K < 1:
        raise ValueError(f"OR-library file: bad problem count {K}")
    for k in range(1, K + 1):
        if pos >= len(v):
            raise ValueError(f"OR-library file: truncated before problem {k}")
        n = v[pos]
        pos += 1
        if n < 1 or pos + columns * n > len(v):
            raise ValueError(f"OR-library file: problem {k} with n={n} is truncated")
        a = np.array(v[pos:pos + columns * n], dtype=np.int64).reshape(n, columns)
        pos += columns * n
        if np.any(a < 0):
            raise ValueError(f"OR-library file: negative value in problem {k}")
        if columns == 3:
            out.append(OrInstance(n, a[:, 0].astype(np.int32), a[:, 1].astype(np.int32),
                                  a[:, 2].astype(np.int32), k=k))
        else:
            out.append(OrInstance(n, a[:, 0].astype(np.int32), a[:, 2].astype(np.int32),
                                  a[:, 3].astype(np.int32), a[:, 1].astype(np.int32),
                                  a[:, 4].astype(np.int32), k=k))
    if pos != len(v):
        raise ValueError(f"OR-library file: {len(v) - pos} trailing values after {K} problems")
    return out


def read_sch(path: str) -> list[OrInstance]:
    with open(path) as f:
        return parse_sch(f.read())


def read_ucddcp(path: str, columns=("P", "M", "alpha", "beta", "gamma")) -> list[OrInstance]:
    """UCDDCP problems, five columns per job in the order `columns`; d = sum P (unrestricted)."""
    want = ("P", "M", "alpha", "beta", "gamma")
    if sorted(columns) != sorted(want):
        raise ValueError(f"columns must be a permutation of {want}")
    with open(path) as f:
        v = parse_sch(f.read(), columns=5)
    out = []
    for inst in v:
        raw = np.stack([inst.P, inst.M, inst.alpha, inst.beta, inst.gamma], axis=1)
        col = {c: raw[:, i] for i, c in enumerate(columns)}
        if np.any(col["M"] > col["P"]):
            raise ValueError(f"problem {inst.k}: M > P")
        out.append(OrInstance(inst.n, col["P"], col["alpha"], col["beta"], col["M"], col["gamma"],
                              d=int(col["P"].sum()), k=inst.k))
    return out


def write_sch(instances: list[OrInstance]) -> str:
    """The sch text of `instances` (p a b per job) -- for tests and for exporting generated sets."""
    lines = [str(len(instances))]
    for inst in instances:
        lines.append(str(inst.n))
        lines += [f"{p} {a} {b}" for p, a, b in zip(inst.P, inst.alpha, inst.beta)]
    return "\n".join(lines) + "\n"


def deviation_pct(z: int, z_best_known: int) -> float:
    """Table II's percentage deviation from the best known solution."""
    return 100.0 * (z - z_best_known) / z_best_known


def to_device(inst: OrInstance, device: int = 0):
    """The libcdd instance (requires the CUDA library)."""
    from . import Instance

    if inst.d is None:
        raise ValueError("choose a due date first (OrInstance.with_h)")
    return Instance(inst.P, inst.alpha, inst.beta, inst.d, inst.M, inst.gamma, device)


def main(argv=None):
    ap = argparse.ArgumentParser(description=__doc__.split("\n")[0])
    ap.add_argument("file")
    ap.add_argument("--k", type=int, default=1, help="problem number in the file (1-based)")
    ap.add_argument("--h", type=float, default=0.4, help="restrictive factor (CDD)")
    ap.add_argument("--ucddcp", action="store_true", help="five-column UCDDCP file, d = sum P")
    ap.add_argument("--chains", type=int, default=65536)
    ap.add_argument("--steps", type=int, default=5000)
    ap.add_argument("--seed", type=int, default=0x5EED0005)
    ap.add_argument("--best-known", type=int, default=None)
    a = ap.parse_args(argv)
    import torch

    from . import best_get, sa_run

    insts = read_ucddcp(a.file) if a.ucddcp else read_sch(a.file)
    if not 1 <= a.k <= len(insts):
        raise SystemExit(f"--k must be in [1, {len(insts)}]")
    inst = insts[a.k - 1] if a.ucddcp else insts[a.k - 1].with_h(a.h)
    dev = to_device(inst)
    problem = "ucddcp" if a.ucddcp else "cdd"
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    sa_run(dev, a.chains, a.steps, problem=problem, seed=a.seed)
    e.record()
    z, perm, g = best_get(dev)
    out = {"file": a.file, "k": a.k, "n": inst.n, "h": None if a.ucddcp else a.h, "d": inst.d,
           "problem": problem, "best": z, "chain": g, "ms": s.elapsed_time(e),
           "sequence": perm.tolist()}
    if a.best_known is not None:
        out["best_known"] = a.best_known
        out["deviation_pct"] = deviation_pct(z, a.best_known)
    print(json.dumps(out))
    return 0


if __name__ == "__main__":
    sys.exit(main())
