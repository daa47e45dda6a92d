"""CPU oracle -- TEST INFRASTRUCTURE ONLY.

ctypes wrapper over ``oracle/oracle.c`` (plain C, written from the paper; see ``oracle.h`` for the
contract and each function's pin status).  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this package.  The product
path (``paper_conf_ipps_awasthillw16_b200``) never imports it and shares no code with it.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_SO = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

CDD, UCDDCP = 0, 1
MOVE_PERT_FY, MOVE_SWAP, MOVE_INSERT, MOVE_WINDOW = 0, 1, 2, 3
TAG_SA_INIT, TAG_SA, TAG_T0, TAG_DPSO_INIT, TAG_DPSO = 0x11, 0x12, 0x13, 0x21, 0x22
WALK_MAX = 64


def build(force: bool = False) -> str:
    """Compile liboracle.so (no FMA contraction, no fast-math)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < max(
        os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "oracle.h"))
    ):
        cmd = ["gcc", "-O2", "-std=gnu11", "-ffp-contract=off", "-fno-fast-math", "-fPIC",
               "-shared", "-Wall", "-Wextra", "-o", _SO + ".tmp", _SRC, "-lm"]
        subprocess.run(cmd, check=True)
        os.replace(_SO + ".tmp", _SO)
    return _SO


class Instance(C.Structure):
    _fields_ = [("n", C.c_int32), ("P", C.c_void_p), ("M", C.c_void_p), ("alpha", C.c_void_p),
                ("beta", C.c_void_p), ("gamma", C.c_void_p), ("d", C.c_int64)]


class Walk(C.Structure):
    _fields_ = [("tau", C.c_int32), ("pe0", C.c_int64), ("pl0", C.c_int64),
                ("first_shift", C.c_int64), ("nsteps", C.c_int32),
                ("pe", C.c_int64 * WALK_MAX), ("pl", C.c_int64 * WALK_MAX),
                ("r", C.c_int32), ("s", C.c_int64)]


class SAParams(C.Structure):
    _fields_ = [("problem", C.c_int32), ("chains", C.c_int64), ("steps", C.c_int64),
                ("mu", C.c_double), ("pert", C.c_int32), ("move", C.c_int32),
                ("seed", C.c_uint64), ("chain_offset", C.c_uint64), ("init", C.c_void_p),
                ("init_ld", C.c_int64)]


class DPSOParams(C.Structure):
    _fields_ = [("problem", C.c_int32), ("particles", C.c_int64), ("iters", C.c_int64),
                ("w", C.c_double), ("c1", C.c_double), ("c2", C.c_double), ("seed", C.c_uint64)]


def _load():
    global _lib
    with _lock:
        if _lib is not None:
            return _lib
        lib = C.CDLL(build())
        vp, i32, i64, u32, u64, dbl = C.c_void_p, C.c_int32, C.c_int64, C.c_uint32, C.c_uint64, C.c_double
        sig = {
            "or_philox4x32_10": (None, [vp, vp, vp]),
            "or_bnd": (u32, [u32, u32]),
            "or_u01": (dbl, [u32]),
            "or_det_exp": (dbl, [dbl]),
            "or_perm_fy": (None, [i32, u64, u32, u64, vp]),
            "or_cdd_eval": (i64, [vp, vp, vp, vp]),
            "or_ucddcp_eval": (i64, [vp, vp, vp, vp]),
            "or_eval_batch": (None, [vp, C.c_int, vp, i64, i64, vp]),
            "or_sa_move": (i32, [i32, i32, i32, u64, u64, u64, vp, vp, vp]),
            "or_sa_neighbour": (None, [i32, i32, i32, vp, vp, vp, vp]),
            "or_t0": (dbl, [vp, i32, u64, i64]),
            "or_sa_chain": (i64, [vp, vp, dbl, u64, vp, vp, vp, vp]),
            "or_sa_run": (None, [vp, vp, dbl, vp, vp, vp, vp]),
            "or_sa_sync": (None, [vp, vp, dbl, i64, vp, vp, vp, vp, vp, vp]),
            "or_dpso_f1": (None, [i32, vp, u32, u32, vp]),
            "or_dpso_f2": (None, [i32, vp, vp, u32, vp]),
            "or_dpso_f3": (None, [i32, vp, vp, u32, u32, vp]),
            "or_dpso_run": (None, [vp, vp, vp, vp, vp, vp]),
        }
        for name, (res, args) in sig.items():
            f = getattr(lib, name)
            f.restype = res
            f.argtypes = args
        _lib = lib
        return lib


def _ptr(a: np.ndarray | None):
    return None if a is None else a.ctypes.data


class Problem:
    """Host copy of one instance (arrays indexed by job id), kept alive for the C struct."""

    def __init__(self, P, alpha, beta, d, M=None, gamma=None):
        self.P = np.ascontiguousarray(P, dtype=np.int32)
        self.alpha = np.ascontiguousarray(alpha, dtype=np.int32)
        self.beta = np.ascontiguousarray(beta, dtype=np.int32)
        self.M = None if M is None else np.ascontiguousarray(M, dtype=np.int32)
        self.gamma = None if gamma is None else np.ascontiguousarray(gamma, dtype=np.int32)
        self.d = int(d)
        self.n = int(self.P.shape[0])
        self.c = Instance(self.n, _ptr(self.P), _ptr(self.M), _ptr(self.alpha), _ptr(self.beta),
                          _ptr(self.gamma), self.d)

    @classmethod
    def from_instance(cls, inst, d=None):
        """From a ``gen.Instance`` (or anything with P, alpha, beta, d[, M, gamma])."""
        return cls(inst.P, inst.alpha, inst.beta, inst.d if d is None else d,
                   getattr(inst, "M", None), getattr(inst, "gamma", None))

    @property
    def ref(self):
        return C.byref(self.c)


# ---------------------------------------------------------------------------------------------
def philox4x32_10(ctr, key) -> np.ndarray:
    c = np.ascontiguousarray(ctr, dtype=np.uint32)
    k = np.ascontiguousarray(key, dtype=np.uint32)
    out = np.zeros(4, dtype=np.uint32)
    _load().or_philox4x32_10(_ptr(c), _ptr(k), _ptr(out))
    return out


def bnd(w: int, m: int) -> int:
    return int(_load().or_bnd(w, m))


def u01(w: int) -> float:
    return float(_load().or_u01(w))


def det_exp(x: float) -> float:
    return float(_load().or_det_exp(float(x)))


def perm_fy(n: int, seed: int, tag: int, ident: int) -> np.ndarray:
    J = np.zeros(n, dtype=np.int16)
    _load().or_perm_fy(n, seed, tag, ident, _ptr(J))
    return J


def cdd_eval(prob: Problem, J, walk: bool = False):
    J = np.ascontiguousarray(J, dtype=np.int16)
    w = Walk()
    Cout = np.zeros(prob.n, dtype=np.int64)
    Z = int(_load().or_cdd_eval(prob.ref, _ptr(J), C.addressof(w), _ptr(Cout)))
    if not walk:
        return Z
    ns = min(w.nsteps, WALK_MAX)
    return Z, {"tau": w.tau, "pe0": w.pe0, "pl0": w.pl0, "first_shift": w.first_shift,
               "nsteps": w.nsteps, "pe": list(w.pe[:ns]), "pl": list(w.pl[:ns]), "r": w.r,
               "s": w.s, "C": Cout}


def ucddcp_eval(prob: Problem, J, detail: bool = False):
    J = np.ascontiguousarray(J, dtype=np.int16)
    X = np.zeros(prob.n, dtype=np.int32)
    Cout = np.zeros(prob.n, dtype=np.int64)
    Z = int(_load().or_ucddcp_eval(prob.ref, _ptr(J), _ptr(X), _ptr(Cout)))
    if Z == -(2**63):
        raise ValueError("UCDDCP requires d >= sum(P) (P:126)")
    return (Z, X, Cout) if detail else Z


def eval_batch(prob: Problem, perms: np.ndarray, problem: int = CDD) -> np.ndarray:
    perms = np.ascontiguousarray(perms, dtype=np.int16)
    B, ld = perms.shape
    out = np.zeros(B, dtype=np.int64)
    _load().or_eval_batch(prob.ref, problem, _ptr(perms), ld, B, _ptr(out))
    return out


def eval_batch_threaded(prob: Problem, perms: np.ndarray, problem: int = CDD,
                        threads: int | None = None) -> np.ndarray:
    """Same as eval_batch, rows split statically over host threads (ctypes drops the GIL)."""
    perms = np.ascontiguousarray(perms, dtype=np.int16)
    B = perms.shape[0]
    threads = threads or os.cpu_count() or 1
    out = np.zeros(B, dtype=np.int64)
    bounds = np.linspace(0, B, threads + 1).astype(np.int64)

    def work(a, b):
        if b > a:
            out[a:b] = eval_batch(prob, perms[a:b], problem)

    ts = [threading.Thread(target=work, args=(bounds[i], bounds[i + 1])) for i in range(threads)]
    [t.start() for t in ts]
    [t.join() for t in ts]
    return out


def sa_move(n, pert, move, seed, g, k):
    q = np.zeros(4, dtype=np.int32)
    s = np.zeros(4, dtype=np.int32)
    u = C.c_double()
    P = _load().or_sa_move(n, pert, move, seed, g, k, _ptr(q), _ptr(s), C.byref(u))
    return q[:P].copy(), s[:P].copy(), u.value


def sa_neighbour(s, move, q, sigma):
    """Alg. 1 line 5: the neighbour of sequence s for the move (q, sigma) drawn by sa_move."""
    s = np.ascontiguousarray(s, dtype=np.int16)
    P = len(q)
    qq = np.zeros(4, dtype=np.int32)
    ss = np.zeros(4, dtype=np.int32)
    qq[:P] = q
    ss[:P] = sigma
    out = np.zeros_like(s)
    _load().or_sa_neighbour(len(s), move, P, _ptr(qq), _ptr(ss), _ptr(s), _ptr(out))
    return out


def t0(prob: Problem, problem: int, seed: int, samples: int = 5000) -> float:
    return float(_load().or_t0(prob.ref, problem, seed, samples))


def sa_params(problem=CDD, chains=1, steps=1000, mu=0.88, pert=4, move=MOVE_PERT_FY, seed=0,
              chain_offset=0, init=None) -> SAParams:
    """init: None (random initial sequences), an int16 [n] array (every chain) or [chains, n]
    (row c for chain c).  The array is kept alive on the returned struct."""
    p = SAParams(problem, chains, steps, mu, pert, move, seed, chain_offset, None, 0)
    if init is not None:
        arr = np.ascontiguousarray(init, dtype=np.int16)
        p._init = arr
        p.init = arr.ctypes.data
        p.init_ld = arr.shape[1] if arr.ndim == 2 else 0
    return p


def sa_chain(prob: Problem, p: SAParams, T0: float, g: int, trace: bool = False):
    n = prob.n
    best = np.zeros(n, dtype=np.int16)
    fin = np.zeros(n, dtype=np.int16)
    fE = C.c_int64()
    tr = np.zeros(p.steps, dtype=np.int64) if trace else None
    Eb = int(_load().or_sa_chain(prob.ref, C.byref(p), T0, g, _ptr(best), C.byref(fE), _ptr(fin),
                                 _ptr(tr)))
    res = {"E_best": Eb, "best": best, "E_final": fE.value, "final": fin}
    if trace:
        res["E_new"] = tr >> 1
        res["accepted"] = (tr & 1).astype(bool)
    return res


def sa_sync(prob: Problem, p: SAParams, T0: float, levels: int):
    """Synchronous SA: p.steps = Markov-chain length M per temperature level."""
    n = prob.n
    bE, bg, bl = C.c_int64(), C.c_uint64(), C.c_int64()
    J = np.zeros(n, dtype=np.int16)
    lE = np.zeros(levels, dtype=np.int64)
    lg = np.zeros(levels, dtype=np.uint64)
    _load().or_sa_sync(prob.ref, C.byref(p), T0, levels, C.byref(bE), C.byref(bg), C.byref(bl),
                       _ptr(J), _ptr(lE), _ptr(lg))
    return {"E_best": bE.value, "g": bg.value, "level": bl.value, "best": J, "level_min_E": lE,
            "level_min_g": lg}


def sa_run(prob: Problem, p: SAParams, T0: float, chain_best: bool = False):
    n = prob.n
    bE = C.c_int64()
    bg = C.c_uint64()
    J = np.zeros(n, dtype=np.int16)
    cb = np.zeros(p.chains, dtype=np.int64) if chain_best else None
    _load().or_sa_run(prob.ref, C.byref(p), T0, C.byref(bE), C.byref(bg), _ptr(J), _ptr(cb))
    res = {"E_best": bE.value, "g": bg.value, "best": J}
    if chain_best:
        res["chain_best"] = cb
    return res


def dpso_f1(p, w1, w2):
    p = np.ascontiguousarray(p, dtype=np.int16)
    out = np.zeros_like(p)
    _load().or_dpso_f1(len(p), _ptr(p), w1, w2, _ptr(out))
    return out


def dpso_f2(lam, pb, wcut):
    lam = np.ascontiguousarray(lam, dtype=np.int16)
    pb = np.ascontiguousarray(pb, dtype=np.int16)
    out = np.zeros_like(lam)
    _load().or_dpso_f2(len(lam), _ptr(lam), _ptr(pb), wcut, _ptr(out))
    return out


def dpso_f3(delta, g, w1, w2):
    delta = np.ascontiguousarray(delta, dtype=np.int16)
    g = np.ascontiguousarray(g, dtype=np.int16)
    out = np.zeros_like(delta)
    _load().or_dpso_f3(len(delta), _ptr(delta), _ptr(g), w1, w2, _ptr(out))
    return out


def dpso_params(problem=CDD, particles=64, iters=100, w=0.5, c1=0.5, c2=0.5, seed=0) -> DPSOParams:
    return DPSOParams(problem, particles, iters, w, c1, c2, seed)


def dpso_run(prob: Problem, p: DPSOParams, trace: bool = False):
    bE = C.c_int64()
    bi = C.c_uint64()
    J = np.zeros(prob.n, dtype=np.int16)
    tr = np.zeros(p.iters, dtype=np.int64) if trace else None
    _load().or_dpso_run(prob.ref, C.byref(p), C.byref(bE), C.byref(bi), _ptr(J), _ptr(tr))
    res = {"E_best": bE.value, "id": bi.value, "best": J}
    if trace:
        res["gbest_trace"] = tr
    return res
