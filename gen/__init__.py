"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds none of the method's arithmetic: it only draws problem data and job sequences.
The OR-library CDD files (Biskup & Feldmann [18]) and the UCDDCP instances of [8]
are not available offline, so instances are generated in the same style:

* p_i ~ U[1,20], alpha_i ~ U[1,10], beta_i ~ U[1,15]     (Biskup-Feldmann ranges, BASELINE.json)
* d = floor(h * sum p) with h in {0.2, 0.4, 0.6, 0.8}    (restrictiveness factor h)
* UCDDCP: x_i = p_i - M_i ~ U[0, floor(p_i/2)], gamma_i ~ U[1,10], d = sum p (unrestricted)
* instance k of a size uses seed k; the job data does not depend on h (as in the OR-library,
  where the four h values share the job data).

Randomness is a counter-based splitmix64 hash of (seed, n, field, index), so every value is
reproducible on any host without depending on numpy's stream policies.
"""
from __future__ import annotations

import dataclasses
import math

import numpy as np

H_VALUES = (0.2, 0.4, 0.6, 0.8)
_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def _mix(x: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser on uint64 arrays (wrapping arithmetic)."""
    with np.errstate(over="ignore"):
        x = x.astype(np.uint64, copy=True)
        x ^= x >> np.uint64(30)
        x *= _M1
        x ^= x >> np.uint64(27)
        x *= _M2
        x ^= x >> np.uint64(31)
    return x


def _words(seed: int, n: int, field: int, count: int) -> np.ndarray:
    """`count` independent uint32 words for stream (seed, n, field)."""
    with np.errstate(over="ignore"):
        base = _mix(np.array([(seed * 0x100000001B3 + n * 0x1F3 + field * 0x9E37) & (2**64 - 1)],
                             dtype=np.uint64))[0]
        x = base + np.arange(1, count + 1, dtype=np.uint64) * _GOLDEN
    return (_mix(x) >> np.uint64(32)).astype(np.uint32)


def _uniform_int(w: np.ndarray, lo: int, hi) -> np.ndarray:
    """lo + floor(w * (hi-lo+1) / 2^32): integers in [lo, hi] (hi may be an array)."""
    span = np.asarray(hi, dtype=np.uint64) - np.uint64(lo) + np.uint64(1)
    return (np.uint64(lo) + ((w.astype(np.uint64) * span) >> np.uint64(32))).astype(np.int32)


@dataclasses.dataclass
class Instance:
    n: int
    P: np.ndarray
    alpha: np.ndarray
    beta: np.ndarray
    M: np.ndarray
    gamma: np.ndarray
    d: int
    seed: int
    h: float | None
    problem: str = "cdd"

    @property
    def sum_p(self) -> int:
        return int(self.P.sum())

    def name(self) -> str:
        hs = "U" if self.h is None else f"{self.h:.1f}"
        return f"{self.problem}-n{self.n}-k{self.seed}-h{hs}"


def cdd_instance(n: int, seed: int, h: float) -> Instance:
    """Biskup-Feldmann-style CDD instance (restrictive for h < 1)."""
    P = _uniform_int(_words(seed, n, 1, n), 1, 20)
    alpha = _uniform_int(_words(seed, n, 2, n), 1, 10)
    beta = _uniform_int(_words(seed, n, 3, n), 1, 15)
    x = _uniform_int(_words(seed, n, 4, n), 0, P // 2)
    gamma = _uniform_int(_words(seed, n, 5, n), 1, 10)
    h_num = int(round(h * 10))
    d = (h_num * int(P.sum())) // 10
    return Instance(n, P, alpha, beta, (P - x).astype(np.int32), gamma, d, seed, h, "cdd")


def ucddcp_instance(n: int, seed: int) -> Instance:
    """UCDDCP instance: the CDD job data plus M_i, gamma_i; d = sum p (unrestricted)."""
    inst = cdd_instance(n, seed, 0.2)
    return dataclasses.replace(inst, d=inst.sum_p, h=None, problem="ucddcp")


def table1() -> Instance:
    """Table I of the paper, d = 16 for the CDD illustration."""
    P = np.array([6, 5, 2, 4, 4], dtype=np.int32)
    M = np.array([5, 5, 2, 3, 3], dtype=np.int32)
    alpha = np.array([7, 9, 6, 9, 3], dtype=np.int32)
    beta = np.array([9, 5, 4, 3, 2], dtype=np.int32)
    gamma = np.array([5, 4, 3, 2, 1], dtype=np.int32)
    return Instance(5, P, alpha, beta, M, gamma, 16, 0, None, "table1")


def ranged_instance(n: int, seed: int, p: tuple, alpha: tuple, beta: tuple, h: float,
                    problem: str = "cdd") -> Instance:
    """Instance with chosen value ranges (inclusive) for edge-case tests: large processing times
    (sum p > 2^16), zero or large penalties (up to 255), d = floor(h * sum p)."""
    P = _uniform_int(_words(seed, n, 21, n), p[0], p[1])
    a = _uniform_int(_words(seed, n, 22, n), alpha[0], alpha[1])
    b = _uniform_int(_words(seed, n, 23, n), beta[0], beta[1])
    x = _uniform_int(_words(seed, n, 24, n), 0, P // 2)
    gamma = _uniform_int(_words(seed, n, 25, n), max(alpha[0], 1), max(alpha[1], 1))
    d = int(math.floor(h * int(P.sum())))
    if problem == "ucddcp":
        d = int(P.sum())
    return Instance(n, P, a, b, (P - x).astype(np.int32), gamma, d, seed, h, problem)


def random_small(n: int, seed: int, pmax: int = 6, wmax: int = 5, h: float | None = None,
                 zero_weights: bool = False) -> Instance:
    """Tiny instances with small values for brute-force pins (optionally zero penalties)."""
    lo = 0 if zero_weights else 1
    P = _uniform_int(_words(seed, n, 11, n), 1, pmax)
    alpha = _uniform_int(_words(seed, n, 12, n), lo, wmax)
    beta = _uniform_int(_words(seed, n, 13, n), lo, wmax)
    x = _uniform_int(_words(seed, n, 14, n), 0, P - 1)
    gamma = _uniform_int(_words(seed, n, 15, n), lo, wmax)
    hh = h if h is not None else float(_uniform_int(_words(seed, n, 16, 1), 0, 13)[0]) / 10.0
    d = int(math.floor(hh * int(P.sum())))
    return Instance(n, P, alpha, beta, (P - x).astype(np.int32), gamma, d, seed, hh, "small")


# --------------------------------------------------------------------------------------------
# Job sequences
# --------------------------------------------------------------------------------------------
def pad_ld(n: int) -> int:
    """Row stride (elements) for int16 sequence batches: a multiple of 16 (32-byte rows, which
    lets the evaluator use 256-bit loads)."""
    return (n + 15) // 16 * 16


def random_perms(batch: int, n: int, seed: int, ld: int | None = None) -> np.ndarray:
    """`batch` uniformly random permutations of 0..n-1 as int16 rows of stride ld (pad = 0)."""
    ld = pad_ld(n) if ld is None else ld
    out = np.zeros((batch, ld), dtype=np.int16)
    chunk = max(1, (1 << 22) // max(n, 1))
    for a in range(0, batch, chunk):
        b = min(batch, a + chunk)
        keys = _mix(np.arange(a * n, b * n, dtype=np.uint64)
                    + np.uint64((seed * 0xD6E8FEB86659FD93) & (2**64 - 1)))
        out[a:b, :n] = np.argsort(keys.reshape(b - a, n), axis=1, kind="stable").astype(np.int16)
    return out


def all_perms(n: int, ld: int | None = None) -> np.ndarray:
    """All n! permutations of 0..n-1 in lexicographic order (n <= 10), int16 rows of stride ld."""
    ld = pad_ld(n) if ld is None else ld
    perms = np.zeros((1, 0), dtype=np.int8)
    for k in range(1, n + 1):
        # perms of range(k): first element f, then perms of the remaining k-1 values
        blocks = []
        for f in range(k):
            rest = np.array([x for x in range(k) if x != f], dtype=np.int8)
            sub = rest[perms] if perms.shape[1] else np.zeros((1, 0), dtype=np.int8)
            blocks.append(np.concatenate([np.full((sub.shape[0], 1), f, dtype=np.int8), sub], axis=1))
        perms = np.concatenate(blocks, axis=0)
    out = np.zeros((perms.shape[0], ld), dtype=np.int16)
    out[:, :n] = perms
    return out


def random_perms_device(batch: int, n: int, seed: int, ld: int | None = None, device="cuda"):
    """Random permutations generated on the device with torch (plumbing for large bench inputs);
    parity checks copy sampled rows back to the host for the oracle."""
    import torch

    ld = pad_ld(n) if ld is None else ld
    out = torch.zeros((batch, ld), dtype=torch.int16, device=device)
    g = torch.Generator(device=device)
    g.manual_seed(seed)
    chunk = max(1, (1 << 26) // max(n, 1))
    for a in range(0, batch, chunk):
        b = min(batch, a + chunk)
        keys = torch.rand((b - a, n), generator=g, device=device)
        out[a:b, :n] = torch.argsort(keys, dim=1).to(torch.int16)
    return out
