"""B200-native hot path of Awasthi, Lässig, Leuschner & Weise, "GPGPU-based Parallel Algorithms for
Scheduling Against Due Date" (IPDPSW 2016): parallel SA chains / a DPSO swarm over the O(n)
optimal-timing routine for CDD and UCDDCP job sequences.

This module is the thin Python binding of ``libcdd.so`` (C-ABI declared in ``include/cdd.h``):
argument marshalling only -- every step of the path runs in the CUDA kernels.  PyTorch provides
device memory (tensors, workspaces), streams and process groups.  There is no CPU fallback: if
the library is missing, importing this package fails.
"""
from __future__ import annotations

import ctypes as C
import os
import re

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.environ.get("CDD_LIB") or os.path.join(_HERE, "libcdd.so")
HEADER = os.path.join(os.path.dirname(_HERE), "include", "cdd.h")

if not os.path.exists(_SO):
    raise ImportError(
        f"libcdd.so not found at {_SO}: build it with `python -c 'import __graft_entry__ as g; "
        f"g.build()'` (there is no CPU fallback)")

_lib = C.CDLL(_SO)

CDD_OK, CDD_EINVAL, CDD_ERANGE, CDD_ENOMEM, CDD_ECUDA, CDD_ESTATE, CDD_EDATA = 0, -1, -2, -3, -4, -5, -6
PROBLEMS = {"cdd": 0, "ucddcp": 1}
MOVES = {"pert_fy": 0, "swap": 1, "insert": 2, "window": 3}


class CddError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"libcdd error {code}: {msg}")
        self.code = code


class SaParams(C.Structure):
    _fields_ = [("problem", C.c_int), ("chains", C.c_int64), ("steps", C.c_int64),
                ("mu", C.c_double), ("T0", C.c_double), ("t0_samples", C.c_int64),
                ("pert", C.c_int32), ("move", C.c_int), ("seed", C.c_uint64),
                ("chain_offset", C.c_uint64), ("trace", C.c_void_p), ("chain_best", C.c_void_p),
                ("chain_final", C.c_void_p), ("T0_out", C.c_void_p), ("T0_in", C.c_void_p),
                ("lanes", C.c_int32), ("init", C.c_void_p), ("init_ld", C.c_int64)]


class SaSyncParams(C.Structure):
    _fields_ = [("problem", C.c_int), ("chains", C.c_int64), ("markov_len", C.c_int64),
                ("levels", C.c_int64), ("mu", C.c_double), ("T0", C.c_double),
                ("t0_samples", C.c_int64), ("pert", C.c_int32), ("move", C.c_int),
                ("seed", C.c_uint64), ("chain_offset", C.c_uint64), ("lanes", C.c_int32),
                ("T0_out", C.c_void_p), ("T0_in", C.c_void_p), ("level_min", C.c_void_p)]


class DpsoParams(C.Structure):
    _fields_ = [("problem", C.c_int), ("particles", C.c_int64), ("iters", C.c_int64),
                ("w", C.c_double), ("c1", C.c_double), ("c2", C.c_double), ("seed", C.c_uint64),
                ("particle_offset", C.c_uint64), ("gbest_trace", C.c_void_p)]


_vp, _i32, _i64, _u64, _sz = C.c_void_p, C.c_int32, C.c_int64, C.c_uint64, C.c_size_t
_SIGS = {
    "cdd_instance_create": (C.c_int, [_i32, _vp, _vp, _vp, _vp, _vp, _i64, C.c_int, C.POINTER(_vp)]),
    "cdd_instance_destroy": (C.c_int, [_vp]),
    "cdd_instance_query": (C.c_int, [_vp, _vp, _vp, _vp, _vp]),
    "cdd_eval_batch": (C.c_int, [_vp, _vp, _i64, _i64, _vp, _vp]),
    "ucddcp_eval_batch": (C.c_int, [_vp, _vp, _i64, _i64, _vp, _vp]),
    "cdd_eval_batch_host": (C.c_int, [_vp, C.c_int, _vp, _i64, _i64, _vp, _vp]),
    "cdd_check": (C.c_int, [_vp, _vp]),
    "cdd_schedule_batch": (C.c_int, [_vp, C.c_int, _vp, _i64, _i64, _vp, _vp, _vp, _vp, _vp]),
    "sa_workspace_size": (_sz, [_vp, C.POINTER(SaParams)]),
    "sa_run": (C.c_int, [_vp, C.POINTER(SaParams), _vp, _sz, _vp]),
    "sa_t0": (C.c_int, [_vp, C.c_int, _u64, _i64, _vp, _vp, _sz, _vp]),
    "sa_layout": (C.c_int, [_vp, C.POINTER(SaParams), _vp, _vp]),
    "sa_sync_workspace_size": (_sz, [_vp, C.POINTER(SaSyncParams)]),
    "sa_sync_run": (C.c_int, [_vp, C.POINTER(SaSyncParams), _vp, _sz, _vp]),
    "sa_sync_level": (C.c_int, [_vp, C.POINTER(SaSyncParams), _vp, _sz, _i64, _vp]),
    "sa_sync_ptrs": (C.c_int, [_vp, C.POINTER(SaSyncParams), _vp, _vp, _vp]),
    "dpso_workspace_size": (_sz, [_vp, C.POINTER(DpsoParams)]),
    "dpso_run": (C.c_int, [_vp, C.POINTER(DpsoParams), _vp, _sz, _vp]),
    "dpso_begin": (C.c_int, [_vp, C.POINTER(DpsoParams), _vp, _sz, _vp]),
    "dpso_iterate": (C.c_int, [_vp, C.POINTER(DpsoParams), _vp, _sz, _i64, _vp]),
    "dpso_gbest_ptrs": (C.c_int, [_vp, C.POINTER(DpsoParams), _vp, _i64, _vp, _vp]),
    "dpso_end": (C.c_int, [_vp, C.POINTER(DpsoParams), _vp, _sz, _vp]),
    "dpso_peer_create": (C.c_int, [_vp, C.c_int, C.c_int, _vp]),
    "dpso_peer_open": (C.c_int, [_vp, _vp]),
    "dpso_peer_reset": (C.c_int, [_vp, _vp]),
    "dpso_peer_destroy": (C.c_int, [_vp]),
    "dpso_run_peer": (C.c_int, [_vp, C.POINTER(DpsoParams), _vp, _sz, _vp]),
    "sa_sync_run_peer": (C.c_int, [_vp, C.POINTER(SaSyncParams), _vp, _sz, _vp]),
    "best_device_ptrs": (C.c_int, [_vp, _vp, _vp]),
    "best_device_ptrs_wide": (C.c_int, [_vp, _vp, _vp]),
    "best_get": (C.c_int, [_vp, _vp, _vp, _vp, _vp]),
    "cdd_last_error": (C.c_char_p, []),
    "cdd_abi_version": (C.c_int, []),
}
for _name, (_res, _args) in _SIGS.items():
    _f = getattr(_lib, _name)
    _f.restype = _res
    _f.argtypes = _args


def header_functions() -> list[str]:
    """Function names declared in include/cdd.h."""
    txt = open(HEADER).read()
    return sorted(set(re.findall(r"^\s*(?:CDD_API\s+)?(?:const\s+)?[a-z_0-9]+\s*\*?\s*([a-z_0-9]+)\s*\(", txt, re.M)))


def _check(rc):
    if rc != CDD_OK:
        raise CddError(rc, _lib.cdd_last_error().decode())


def _stream(stream):
    if stream is None:
        import torch

        return torch.cuda.current_stream().cuda_stream
    return getattr(stream, "cuda_stream", stream)


def _dptr(t):
    return None if t is None else t.data_ptr()


def _i32arr(x):
    return None if x is None else np.ascontiguousarray(x, dtype=np.int32)


class Instance:
    """A problem instance resident on one GPU (wraps ``cdd_instance*``)."""

    def __init__(self, P, alpha, beta, d, M=None, gamma=None, device=0):
        P, alpha, beta, M, gamma = map(_i32arr, (P, alpha, beta, M, gamma))
        self.n = int(P.shape[0])
        self.d = int(d)
        self.device = int(device)
        h = _vp()
        _check(_lib.cdd_instance_create(self.n, P.ctypes.data, alpha.ctypes.data, beta.ctypes.data,
                                        None if M is None else M.ctypes.data,
                                        None if gamma is None else gamma.ctypes.data,
                                        self.d, self.device, C.byref(h)))
        self._h = h
        self.sum_p = int(P.sum())
        self.wide = self.query()["generic"]

    @classmethod
    def from_gen(cls, inst, device=0):
        return cls(inst.P, inst.alpha, inst.beta, inst.d, inst.M, inst.gamma, device)

    def query(self):
        """cdd_instance_query: dict(n, d, sum_p, has_ucddcp, unrestricted, generic, ucddcp_generic,
        small_weights)."""
        n, d, sp, fl = C.c_int32(), C.c_int64(), C.c_int64(), C.c_int32()
        _check(_lib.cdd_instance_query(self.handle, C.byref(n), C.byref(d), C.byref(sp), C.byref(fl)))
        return dict(n=n.value, d=d.value, sum_p=sp.value, has_ucddcp=bool(fl.value & 1),
                    unrestricted=bool(fl.value & 2), generic=bool(fl.value & 4),
                    ucddcp_generic=bool(fl.value & 8), small_weights=bool(fl.value & 16))

    @property
    def handle(self):
        if self._h is None:
            raise CddError(CDD_EINVAL, "instance destroyed")
        return self._h

    def destroy(self):
        if getattr(self, "_h", None) is not None:
            _lib.cdd_instance_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass


def cdd_instance_create(P, alpha, beta, d, M=None, gamma=None, device=0) -> Instance:
    return Instance(P, alpha, beta, d, M, gamma, device)


def cdd_instance_destroy(inst: Instance) -> None:
    inst.destroy()


def _eval(fn, inst, perms, out, stream):
    import torch

    assert perms.dtype == torch.int16 and perms.dim() == 2 and perms.is_cuda
    assert perms.stride(1) == 1
    B, ld = perms.shape[0], perms.stride(0)
    if out is None:
        out = torch.empty(B, dtype=torch.int64, device=perms.device)
    _check(fn(inst.handle, perms.data_ptr(), ld, B, out.data_ptr(), _stream(stream)))
    return out


def cdd_eval_batch(inst: Instance, perms, out=None, stream=None):
    """out[b] = optimal CDD penalty of sequence perms[b, :n] (device int16 [B, ld])."""
    return _eval(_lib.cdd_eval_batch, inst, perms, out, stream)


def ucddcp_eval_batch(inst: Instance, perms, out=None, stream=None):
    """out[b] = optimal UCDDCP penalty of sequence perms[b, :n]."""
    return _eval(_lib.ucddcp_eval_batch, inst, perms, out, stream)


def cdd_schedule_batch(inst: Instance, perms, problem="cdd", stream=None):
    """Optimal schedules of device int16 [B, ld] sequences: dict of device tensors C [B, n] (int64),
    X [B, n] (int32, UCDDCP), start [B], penalty [B]."""
    import torch

    assert perms.dtype == torch.int16 and perms.dim() == 2 and perms.is_cuda and perms.stride(1) == 1
    B, ld = perms.shape[0], perms.stride(0)
    dev = perms.device
    out = {"C": torch.empty((B, inst.n), dtype=torch.int64, device=dev),
           "start": torch.empty(B, dtype=torch.int64, device=dev),
           "penalty": torch.empty(B, dtype=torch.int64, device=dev)}
    if problem == "ucddcp":
        out["X"] = torch.empty((B, inst.n), dtype=torch.int32, device=dev)
    _check(_lib.cdd_schedule_batch(inst.handle, PROBLEMS[problem], perms.data_ptr(), ld, B,
                                   out["C"].data_ptr(), _dptr(out.get("X")), out["start"].data_ptr(),
                                   out["penalty"].data_ptr(), _stream(stream)))
    return out


def schedule_get(inst: Instance, perm, problem="cdd"):
    """Optimal schedule of one host sequence (e.g. best_get's): numpy C (int64 [n]), X (int32 [n]
    or None), start, penalty.  Synchronous."""
    import torch

    ld = (inst.n + 7) // 8 * 8
    p = torch.zeros((1, ld), dtype=torch.int16)
    p[0, :inst.n] = torch.from_numpy(np.ascontiguousarray(perm, dtype=np.int16))
    out = cdd_schedule_batch(inst, p.to(torch.device("cuda", inst.device)), problem)
    torch.cuda.synchronize(inst.device)
    X = out["X"][0].cpu().numpy() if "X" in out else None
    return out["C"][0].cpu().numpy(), X, int(out["start"][0].item()), int(out["penalty"][0].item())


def cdd_eval_batch_host(inst: Instance, perms: np.ndarray, problem="cdd", out=None, stream=None):
    """End-to-end evaluation of HOST sequences (int16 [B, ld]) into a host int64 array."""
    perms = np.ascontiguousarray(perms, dtype=np.int16) if isinstance(perms, np.ndarray) else perms
    if isinstance(perms, np.ndarray):
        B, ld = perms.shape
        pptr = perms.ctypes.data
    else:  # pinned torch CPU tensor
        B, ld = perms.shape
        pptr = perms.data_ptr()
    if out is None:
        out = np.empty(B, dtype=np.int64)
    optr = out.ctypes.data if isinstance(out, np.ndarray) else out.data_ptr()
    _check(_lib.cdd_eval_batch_host(inst.handle, PROBLEMS[problem], pptr, ld, B, optr,
                                    _stream(stream)))
    return out


def cdd_check(inst: Instance, stream=None) -> None:
    _check(_lib.cdd_check(inst.handle, _stream(stream)))


def _sa_params(problem, chains, steps, mu, T0, t0_samples, pert, move, seed, chain_offset,
               trace=None, chain_best=None, chain_final=None, T0_out=None, T0_in=None, lanes=0):
    return SaParams(PROBLEMS[problem], int(chains), int(steps), float(mu), float(T0),
                    int(t0_samples), int(pert), MOVES[move], int(seed) & (2**64 - 1),
                    int(chain_offset), _dptr(trace), _dptr(chain_best), _dptr(chain_final),
                    _dptr(T0_out), _dptr(T0_in), int(lanes))


def sa_workspace_size(inst: Instance, **kw) -> int:
    p = _sa_params(**kw)
    return int(_lib.sa_workspace_size(inst.handle, C.byref(p)))


def sa_run(inst: Instance, chains: int, steps: int, problem="cdd", mu=0.88, T0=0.0,
           t0_samples=5000, pert=4, move="pert_fy", seed=0, chain_offset=0, trace=False,
           chain_best=False, chain_final=False, stream=None, workspace=None, T0_dev=None, lanes=0,
           init=None):
    """Asynchronous parallel SA (Alg. 1): `chains` independent chains of `steps` iterations,
    reduced to the best (penalty, chain) into the instance's best buffers.  Returns the optional
    per-chain device tensors (and the T0 used) without synchronising.  `lanes`: threads per
    chain (0 automatic, 32, 16, 8, 4) -- a speed knob only, results are identical.  `init`:
    optional device int16 initial sequences s0 -- [n] for every chain or [chains, ld]
    (row c for local chain c); None: each chain's own random sequence."""
    import torch

    dev = torch.device("cuda", inst.device)
    res = {"T0": torch.empty(1, dtype=torch.float64, device=dev)}
    if trace:
        res["trace"] = torch.empty((chains, steps), dtype=torch.int64, device=dev)
    if chain_best:
        res["chain_best"] = torch.empty(chains, dtype=torch.int64, device=dev)
    if chain_final:
        res["chain_final"] = torch.empty(chains, dtype=torch.int64, device=dev)
    p = _sa_params(problem, chains, steps, mu, T0, t0_samples, pert, move, seed, chain_offset,
                   res.get("trace"), res.get("chain_best"), res.get("chain_final"), res["T0"],
                   T0_dev, lanes)
    if init is not None:
        assert init.dtype == torch.int16 and init.is_cuda and init.stride(-1) == 1
        assert (init.dim() == 1 and init.shape[0] >= inst.n) or (
            init.dim() == 2 and init.shape[0] >= chains and init.shape[1] >= inst.n)
        p.init = init.data_ptr()
        p.init_ld = 0 if init.dim() == 1 else init.stride(0)
        res["init"] = init  # keep alive until the (asynchronous) run is done with it
    need = int(_lib.sa_workspace_size(inst.handle, C.byref(p)))
    if need == 0:
        _check(_lib.sa_run(inst.handle, C.byref(p), None, 0, None))  # raises with the reason
    if workspace is None or workspace.numel() < need:
        workspace = torch.empty(need, dtype=torch.uint8, device=dev)
    res["workspace"] = workspace
    _check(_lib.sa_run(inst.handle, C.byref(p), workspace.data_ptr(), need, _stream(stream)))
    return res


def sa_layout(inst: Instance, chains: int, problem="cdd", lanes=0):
    """(threads per chain, positions per thread) that sa_run uses for these arguments."""
    p = _sa_params(problem, chains, 1, 0.88, 1.0, 0, 4, "pert_fy", 0, 0, lanes=lanes)
    g, e = C.c_int32(), C.c_int32()
    _check(_lib.sa_layout(inst.handle, C.byref(p), C.byref(g), C.byref(e)))
    return g.value, e.value


def sa_t0(inst: Instance, problem="cdd", seed=0, samples=5000, stream=None):
    """T0 rule of P:192 on the device: population std of `samples` random sequences."""
    import torch

    dev = torch.device("cuda", inst.device)
    p = _sa_params(problem, 1, 0, 0.88, 0.0, samples, 4, "pert_fy", seed, 0)
    need = int(_lib.sa_workspace_size(inst.handle, C.byref(p)))
    ws = torch.empty(max(need, 1), dtype=torch.uint8, device=dev)
    T0 = torch.empty(1, dtype=torch.float64, device=dev)
    _check(_lib.sa_t0(inst.handle, PROBLEMS[problem], int(seed), int(samples), T0.data_ptr(),
                      ws.data_ptr(), need, _stream(stream)))
    return T0


class SaSync:
    """Synchronous SA on one GPU: `run()` does every level; `level(j)` and
    `exchange_tensors()` let a caller share s^min across GPUs between levels."""

    def __init__(self, inst: Instance, chains: int, markov_len: int, levels: int, problem="cdd",
                 mu=0.88, T0=0.0, t0_samples=5000, pert=4, move="pert_fy", seed=0,
                 chain_offset=0, lanes=0, level_min=True, T0_dev=None):
        import torch

        self.inst = inst
        dev = torch.device("cuda", inst.device)
        self.T0 = torch.empty(1, dtype=torch.float64, device=dev)
        self.level_min = torch.empty(levels, dtype=torch.int64, device=dev) if level_min else None
        self.p = SaSyncParams(PROBLEMS[problem], int(chains), int(markov_len), int(levels), float(mu),
                              float(T0), int(t0_samples), int(pert), MOVES[move],
                              int(seed) & (2**64 - 1), int(chain_offset), int(lanes),
                              self.T0.data_ptr(), _dptr(T0_dev), _dptr(self.level_min))
        need = int(_lib.sa_sync_workspace_size(inst.handle, C.byref(self.p)))
        if need == 0:
            _check(_lib.sa_sync_run(inst.handle, C.byref(self.p), None, 0, None))  # raises
        self.ws = torch.empty(need, dtype=torch.uint8, device=dev)

    def run(self, stream=None):
        _check(_lib.sa_sync_run(self.inst.handle, C.byref(self.p), self.ws.data_ptr(),
                                self.ws.numel(), _stream(stream)))
        return self

    def run_peer(self, stream=None):
        """All levels with s^min exchanged across ranks inside the kernels (sa_sync_run_peer)."""
        _check(_lib.sa_sync_run_peer(self.inst.handle, C.byref(self.p), self.ws.data_ptr(),
                                     self.ws.numel(), _stream(stream)))
        return self

    def level(self, j: int, stream=None):
        _check(_lib.sa_sync_level(self.inst.handle, C.byref(self.p), self.ws.data_ptr(),
                                  self.ws.numel(), int(j), _stream(stream)))

    def exchange_tensors(self):
        """(key int64 [1], s^min int16 [n]) device views for the between-level exchange."""
        k, q = _vp(), _vp()
        _check(_lib.sa_sync_ptrs(self.inst.handle, C.byref(self.p), self.ws.data_ptr(),
                                 C.byref(k), C.byref(q)))
        return (_device_view(k.value, (1,), "<i8", self.inst.device),
                _device_view(q.value, (self.inst.n,), "<i2", self.inst.device))


def sa_sync_run(inst: Instance, chains: int, markov_len: int, levels: int, **kw) -> SaSync:
    """Synchronous SA on one GPU; the best-ever state goes to the instance's best buffers."""
    return SaSync(inst, chains, markov_len, levels, **kw).run()


class Dpso:
    """A DPSO swarm on one GPU (Alg. 2, eq. (3)).  `run()` does the whole single-GPU run; the
    stepping methods let a caller exchange the swarm best across GPUs between iterations."""

    def __init__(self, inst: Instance, particles: int, iters: int, problem="cdd", w=0.5, c1=0.5,
                 c2=0.5, seed=0, particle_offset=0, trace=False):
        import torch

        self.inst = inst
        dev = torch.device("cuda", inst.device)
        self.trace = torch.empty(max(iters, 1), dtype=torch.int64, device=dev) if trace else None
        self.p = DpsoParams(PROBLEMS[problem], int(particles), int(iters), float(w), float(c1),
                            float(c2), int(seed), int(particle_offset), _dptr(self.trace))
        need = int(_lib.dpso_workspace_size(inst.handle, C.byref(self.p)))
        if need == 0:
            _check(_lib.dpso_run(inst.handle, C.byref(self.p), None, 0, None))
        self.ws = torch.empty(need, dtype=torch.uint8, device=dev)
        self.iters = int(iters)

    def _args(self):
        return self.inst.handle, C.byref(self.p), self.ws.data_ptr(), self.ws.numel()

    def run(self, stream=None):
        _check(_lib.dpso_run(*self._args(), _stream(stream)))
        return self

    def run_peer(self, stream=None):
        """The whole run with the swarm best exchanged inside the kernels through the instance's
        peer exchange (dpso_peer_create / open / reset; see dist.dpso_run_distributed)."""
        _check(_lib.dpso_run_peer(*self._args(), _stream(stream)))
        return self

    def begin(self, stream=None):
        _check(_lib.dpso_begin(*self._args(), _stream(stream)))

    def iterate(self, t, stream=None):
        h, p, w, nb = self._args()
        _check(_lib.dpso_iterate(h, p, w, nb, int(t), _stream(stream)))

    def end(self, stream=None):
        _check(_lib.dpso_end(*self._args(), _stream(stream)))

    def gbest_tensors(self, t):
        """Torch views of the swarm-best key (int64 [1]) and sequence (int16 [n]) iteration t reads."""
        import torch

        key = _vp()
        perm = _vp()
        _check(_lib.dpso_gbest_ptrs(self.inst.handle, C.byref(self.p), self.ws.data_ptr(), int(t),
                                    C.byref(key), C.byref(perm)))
        dev = torch.device("cuda", self.inst.device)
        return (torch.as_tensor(_CudaArray(key.value, (1,), "<i8"), device=dev),
                torch.as_tensor(_CudaArray(perm.value, (self.inst.n,), "<i2"), device=dev))


def dpso_run(inst: Instance, particles: int, iters: int, problem="cdd", w=0.5, c1=0.5, c2=0.5,
             seed=0, trace=False, stream=None):
    """Discrete PSO (Alg. 2, eq. (3)) on one GPU; best into the instance's best buffers."""
    sw = Dpso(inst, particles, iters, problem, w, c1, c2, seed, 0, trace).run(stream)
    return {"gbest_trace": sw.trace, "workspace": sw.ws, "swarm": sw}


IPC_HANDLE_BYTES = 64


def dpso_peer_create(inst: Instance, world: int, rank: int) -> bytes:
    """This rank's exchange region; returns its CUDA IPC handle (IPC_HANDLE_BYTES bytes)."""
    h = (C.c_uint8 * IPC_HANDLE_BYTES)()
    _check(_lib.dpso_peer_create(inst.handle, int(world), int(rank), h))
    return bytes(h)


def dpso_peer_open(inst: Instance, handles: list) -> None:
    """Map every other rank's region (handles in rank order)."""
    buf = b"".join(handles)
    arr = (C.c_uint8 * len(buf)).from_buffer_copy(buf)
    _check(_lib.dpso_peer_open(inst.handle, arr))


def dpso_peer_reset(inst: Instance, stream=None) -> None:
    _check(_lib.dpso_peer_reset(inst.handle, _stream(stream)))


def dpso_peer_destroy(inst: Instance) -> None:
    _check(_lib.dpso_peer_destroy(inst.handle))


def best_device_ptrs(inst: Instance):
    key = _vp()
    perm = _vp()
    _check(_lib.best_device_ptrs(inst.handle, C.byref(key), C.byref(perm)))
    return key.value, perm.value


class _CudaArray:
    def __init__(self, ptr, shape, typestr):
        self.__cuda_array_interface__ = {"shape": shape, "typestr": typestr, "data": (ptr, False),
                                         "version": 3, "strides": None}


def _device_view(ptr, shape, typestr, device):
    import torch

    return torch.as_tensor(_CudaArray(ptr, shape, typestr), device=torch.device("cuda", device))


def best_device_tensors_wide(inst: Instance):
    """Generic-path instances: torch views of the device {penalty, global id} (int64 [2]) and the
    int16 [n] best sequence."""
    kp, pp = _vp(), _vp()
    _check(_lib.best_device_ptrs_wide(inst.handle, C.byref(kp), C.byref(pp)))
    return (_device_view(kp.value, (2,), "<i8", inst.device),
            _device_view(pp.value, (inst.n,), "<i2", inst.device))


def best_device_tensors(inst: Instance):
    """Torch views (no copy) of the instance's best buffers: packed int64 key [1], int16 [n]."""
    import torch

    kp, pp = best_device_ptrs(inst)
    dev = torch.device("cuda", inst.device)
    key = torch.as_tensor(_CudaArray(kp, (1,), "<i8"), device=dev)
    perm = torch.as_tensor(_CudaArray(pp, (inst.n,), "<i2"), device=dev)
    return key, perm


def best_get(inst: Instance, stream=None):
    """(penalty, sequence as np.int16[n], global chain/particle id) -- synchronises."""
    pen = C.c_int64()
    gid = C.c_uint64()
    perm = np.zeros(inst.n, dtype=np.int16)
    _check(_lib.best_get(inst.handle, C.byref(pen), perm.ctypes.data, C.byref(gid), _stream(stream)))
    return pen.value, perm, gid.value


def abi_version() -> int:
    return int(_lib.cdd_abi_version())
