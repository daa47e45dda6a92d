"""Independent brute-force solvers used to pin the oracle (test helpers; no oracle code).

* ``shift_bf``  -- CDD for a fixed sequence: min over integer start s in [0, max(d,0)] of the
  no-idle objective eq. (1).  Complete: for s > d every job is tardy and the cost grows.
* ``dp_schedule`` -- CDD/UCDDCP for a fixed sequence by dynamic programming over integer completion
  times, idle time ALLOWED and every integer compression X_i in [0, P_i - M_i] tried.  It is the LP
  of P:65-69 for fixed delta_ij solved exhaustively on the integer grid (so it does not assume the
  no-idle property of [9] nor Property 2 of [8]).
* ``lp_schedule`` -- the same LP solved by scipy's HiGHS in continuous variables.
"""
from __future__ import annotations

import itertools

import numpy as np


def objective(P, a, b, d, J, s, X=None, g=None):
    """eq. (1)/(2) for the no-idle schedule starting at s with processing times P - X."""
    C = s
    Z = 0
    for k, j in enumerate(J):
        x = 0 if X is None else int(X[k])
        C += int(P[j]) - x
        Z += int(a[j]) * max(0, d - C) + int(b[j]) * max(0, C - d)
        if X is not None:
            Z += int(g[j]) * x
    return Z


def shift_bf(P, a, b, d, J):
    return min(objective(P, a, b, d, J, s) for s in range(0, max(int(d), 0) + 1))


def dp_schedule(P, a, b, d, J, M=None, g=None, horizon=None):
    """min over integer completion times (idle allowed) and integer X of eq. (1)/(2)."""
    d = int(d)
    H = horizon if horizon is not None else max(d, 0) + int(sum(int(P[j]) for j in J)) + 2
    INF = float("inf")
    prev_best = np.zeros(H + 1)  # f(0, t) = 0 for every t >= 0 (machine free from time 0)
    for j in J:
        xs = [0] if M is None else range(0, int(P[j]) - int(M[j]) + 1)
        cur = np.full(H + 1, INF)
        for t in range(H + 1):
            cost_t = int(a[j]) * max(0, d - t) + int(b[j]) * max(0, t - d)
            for x in xs:
                pt = int(P[j]) - x
                if t - pt < 0:
                    continue
                c = prev_best[t - pt] + cost_t + (0 if M is None else int(g[j]) * x)
                if c < cur[t]:
                    cur[t] = c
        prev_best = np.minimum.accumulate(cur)  # best over completion times <= t
    return int(prev_best[H])


def lp_schedule(P, a, b, d, J, M=None, g=None):
    """LP of P:67 for a fixed sequence, continuous variables, solved with scipy HiGHS."""
    from scipy.optimize import linprog

    n = len(J)
    # variables: C (n), E (n), T (n), X (n)
    nv = 4 * n
    cost = np.zeros(nv)
    for k, j in enumerate(J):
        cost[n + k] = a[j]
        cost[2 * n + k] = b[j]
        cost[3 * n + k] = 0 if M is None else g[j]
    A, ub = [], []

    def row():
        return np.zeros(nv)

    for k, j in enumerate(J):
        r = row(); r[n + k] = -1; r[k] = -1; A.append(r); ub.append(-d)      # E_k >= d - C_k
        r = row(); r[2 * n + k] = -1; r[k] = 1; A.append(r); ub.append(d)    # T_k >= C_k - d
        if k == 0:
            r = row(); r[0] = -1; r[3 * n] = -1; A.append(r); ub.append(-P[j])  # C_1 >= P - X
        else:
            r = row(); r[k] = -1; r[k - 1] = 1; r[3 * n + k] = -1; A.append(r); ub.append(-P[j])
    bounds = [(None, None)] * n + [(0, None)] * (2 * n)
    for k, j in enumerate(J):
        bounds.append((0, 0) if M is None else (0, int(P[j]) - int(M[j])))
    res = linprog(cost, A_ub=np.array(A), b_ub=np.array(ub), bounds=bounds, method="highs")
    assert res.status == 0, res.message
    return res.fun


def v_shaped(P, a, b, J) -> bool:
    """Early part by P/alpha non-increasing, optional straddling job, tardy part by P/beta
    non-decreasing (the V-shape of optimal CDD schedules, BASELINE.json north_star (2))."""
    n = len(J)

    def early_ok(seq):
        return all(P[x] * a[y] >= P[y] * a[x] for x, y in zip(seq, seq[1:]))

    def tardy_ok(seq):
        return all(P[x] * b[y] <= P[y] * b[x] for x, y in zip(seq, seq[1:]))

    for k in range(n + 1):
        if not early_ok(J[:k]):
            break
        if tardy_ok(J[k:]) or (k < n and tardy_ok(J[k + 1:])):
            return True
    return False


def all_sequences(n):
    return [list(p) for p in itertools.permutations(range(n))]


def breakpoint_bf(P, a, b, d, J, X=None, g=None):
    """Exact (Python integers, any magnitude) min over integer starts s >= 0 of the no-idle
    objective eq. (1)/(2).  The objective is convex piecewise linear in s with breakpoints where
    some job completes exactly at d, so the minimum over s in [0, inf) is attained at s = 0 or at
    one of the starts s = d - C_k >= 0 (C_k = completion time of position k when starting at 0)."""
    d = int(d)
    C, cands = 0, {0}
    for k, j in enumerate(J):
        C += int(P[j]) - (0 if X is None else int(X[k]))
        if d - C >= 0:
            cands.add(d - C)
    return min(objective(P, a, b, d, J, s, X, g) for s in cands)


def ucddcp_vertex_bf(P, a, b, d, J, M, g):
    """Exact UCDDCP for a fixed sequence with d >= sum P: every compression vector with X_k in
    {0, P_k - M_k} (the LP's vertices in X: for a fixed start the objective is linear in each X_k
    between two breakpoints, so an optimum exists at an extreme compression -- checked against the
    integer DP on small values) times the exact start enumeration."""
    n = len(J)
    full = [int(P[j]) - int(M[j]) for j in J]
    best = None
    for mask in range(1 << n):
        X = [full[k] if (mask >> k) & 1 else 0 for k in range(n)]
        z = breakpoint_bf(P, a, b, d, J, X, g)
        best = z if best is None or z < best else best
    return best
