"""Oracle B -- TEST INFRASTRUCTURE ONLY.

The literal assignment LP of Eqs. 2-6 (Table 1) for a
fixed placement x, in exact rational arithmetic (``fractions.Fraction``), solved
by a dense two-phase simplex with Bland's rule.  Nothing is reduced by hand:
every y_{d,q} and z_{d,q} of Table 1 is a variable, and each constraint is
written as the paper states it, with x fixed:

  Eq. 2   sum_d y_{d,q} <= 1                                   for all q
  Eq. 3   sum_m sum_d B_{m,q} x_{d,m} y_{d,q} = sum_d y_{d,q}  for all q
  y       y_{d,q} <= 1   (y in [0, 1])
  Eq. 4   sum_q z_{d,q} <= sum_q y_{d,q} s_q                   for all d
  Eq. 5   z_{d,q} <= sum_m P_{d,m,q} x_{d,m}                   for all d, q
  Eq. 6   relaxed by reading C1: stage 1 maximises served = sum_{d,q} z_{d,q};
          stage 2 fixes served at its optimum and maximises
  Eq. 7   sum_q a_q,  a_q = sum_m A_m sum_d x_{d,m} z_{d,q}   (reading C2)

It shares nothing with the CUDA path or with oracle.c's vertex enumeration.
"""

from __future__ import annotations

from fractions import Fraction as Fr

import numpy as np


class Unbounded(Exception):
    pass


class Infeasible(Exception):
    pass


def _pivot(T, basis, r, c):
    piv = T[r][c]
    T[r] = [v / piv for v in T[r]]
    row = T[r]
    for i in range(len(T)):
        if i != r:
            f = T[i][c]
            if f != 0:
                T[i] = [a - f * b for a, b in zip(T[i], row)]
    basis[r] = c


def _optimize(T, basis, obj, allowed):
    """Primal simplex, Bland's rule (smallest entering and leaving index)."""
    n = len(T[0]) - 1
    while True:
        cb = [obj[b] for b in basis]
        enter = None
        for j in range(n):
            if not allowed[j] or j in basis:
                continue
            rc = obj[j] - sum(cb[i] * T[i][j] for i in range(len(T)) if T[i][j] != 0)
            if rc > 0:
                enter = j
                break
        if enter is None:
            return
        best = None
        for i in range(len(T)):
            if T[i][enter] > 0:
                ratio = T[i][-1] / T[i][enter]
                if best is None or ratio < best[0] or (ratio == best[0] and basis[i] < basis[best[1]]):
                    best = (ratio, i)
        if best is None:
            raise Unbounded()
        _pivot(T, basis, best[1], enter)


def _presolve_zero_fixed(nx, A_ub, b_ub, A_eq, b_eq):
    """Generic LP presolve (nothing specific to Eqs. 2-6): with x >= 0, a row
    whose nonzero coefficients all have one sign and whose right-hand side is
    0 -- an equality, or a <= row with positive coefficients -- forces every
    variable in it to 0.  Repeated to a fixed point; returns the set of fixed
    variables."""
    fixed = set()
    changed = True
    while changed:
        changed = False
        rows = [(a, b, True) for a, b in zip(A_eq, b_eq)] + [(a, b, False) for a, b in zip(A_ub, b_ub)]
        for a, b, eq in rows:
            if b != 0:
                continue
            nz = [j for j in range(nx) if a[j] != 0 and j not in fixed]
            if not nz:
                continue
            pos = all(a[j] > 0 for j in nz)
            neg = all(a[j] < 0 for j in nz)
            if pos or (eq and neg):
                fixed.update(nz)
                changed = True
    return fixed


def lp_max(c, A_ub, b_ub, A_eq, b_eq, presolve=False):
    """max c.x  s.t. A_ub x <= b_ub, A_eq x = b_eq, x >= 0 (all Fractions).
    Returns (value, x).  presolve=True first removes the variables that
    _presolve_zero_fixed fixes at 0 (and rows left empty, after checking
    them), then solves the rest with the same simplex."""
    if presolve:
        nx = len(c)
        fixed = _presolve_zero_fixed(nx, A_ub, b_ub, A_eq, b_eq)
        keep = [j for j in range(nx) if j not in fixed]
        red = lambda a: [a[j] for j in keep]  # noqa: E731
        rub, rbu, req, rbe = [], [], [], []
        for a, b in zip(A_ub, b_ub):
            if any(a[j] != 0 for j in keep):
                rub.append(red(a)); rbu.append(b)
            elif b < 0:
                raise Infeasible()
        for a, b in zip(A_eq, b_eq):
            if any(a[j] != 0 for j in keep):
                req.append(red(a)); rbe.append(b)
            elif b != 0:
                raise Infeasible()
        val, xr = lp_max(red(c), rub, rbu, req, rbe)
        x = [Fr(0)] * nx
        for j, v in zip(keep, xr):
            x[j] = v
        return val, x
    nx = len(c)
    rows = []  # (coeffs over x, slack sign or None, rhs)
    for a, b in zip(A_ub, b_ub):
        rows.append((list(a), 1, b))
    for a, b in zip(A_eq, b_eq):
        rows.append((list(a), None, b))
    m = len(rows)
    n_slack = sum(1 for r in rows if r[1] is not None)
    # columns: x | slacks | artificials (one per row) | rhs
    ncol = nx + n_slack + m
    T = []
    basis = []
    si = 0
    for i, (a, sgn, b) in enumerate(rows):
        row = [Fr(0)] * (ncol + 1)
        for j, v in enumerate(a):
            row[j] = Fr(v)
        if sgn is not None:
            row[nx + si] = Fr(1)
            si += 1
        row[-1] = Fr(b)
        if row[-1] < 0:
            row = [-v for v in row]
        row[nx + n_slack + i] = Fr(1)
        T.append(row)
        basis.append(nx + n_slack + i)
    # phase 1: maximise -sum(artificials)
    obj1 = [Fr(0)] * (nx + n_slack) + [Fr(-1)] * m
    _optimize(T, basis, obj1, [True] * ncol)
    if sum(T[i][-1] for i in range(m) if basis[i] >= nx + n_slack) != 0:
        raise Infeasible()
    # drive remaining (zero-valued) artificials out of the basis where possible
    for i in range(m):
        if basis[i] >= nx + n_slack:
            for j in range(nx + n_slack):
                if T[i][j] != 0:
                    _pivot(T, basis, i, j)
                    break
    allowed = [True] * (nx + n_slack) + [False] * m
    obj2 = [Fr(v) for v in c] + [Fr(0)] * (n_slack + m)
    _optimize(T, basis, obj2, allowed)
    x = [Fr(0)] * ncol
    for i, b in enumerate(basis):
        x[b] = T[i][-1]
    val = sum(Fr(cj) * x[j] for j, cj in enumerate(c))
    return val, x[:nx]


def literal_assignment_lp(P_tm, acc_m, V, device_type, option, demand, presolve=False):
    """Solve Eqs. 2-6 (+ reading C1 lexicographic objective) for placement x
    given as option[d] (0 idle, else 1 + variant index m).  Returns
    (served, accsum, z[d][q]) with Fractions.  presolve=True hands the same
    constraint rows to lp_max's generic zero-fixing presolve (needed for
    c2/c3-sized placements: the dense tableau of D*Q*2 columns is otherwise
    too slow in Fractions)."""
    V = list(map(int, V))
    Q = len(V)
    D = len(option)
    fam = [q for q in range(Q) for _ in range(V[q])]
    M = len(fam)
    x = [[1 if option[d] == m + 1 else 0 for m in range(M)] for d in range(D)]
    assert all(sum(x[d]) <= 1 for d in range(D))  # Eq. 1
    B = [[1 if fam[m] == q else 0 for q in range(Q)] for m in range(M)]
    Pdmq = lambda d, m, q: int(P_tm[device_type[d]][m]) if B[m][q] else 0
    # variable layout: y[d][q] at d*Q+q, z[d][q] at D*Q + d*Q+q
    ny = D * Q
    nv = 2 * D * Q
    Y = lambda d, q: d * Q + q
    Z = lambda d, q: ny + d * Q + q
    A_ub, b_ub, A_eq, b_eq = [], [], [], []
    for q in range(Q):  # Eq. 2
        a = [0] * nv
        for d in range(D):
            a[Y(d, q)] = 1
        A_ub.append(a); b_ub.append(1)
    for q in range(Q):  # Eq. 3
        a = [0] * nv
        for d in range(D):
            a[Y(d, q)] += sum(B[m][q] * x[d][m] for m in range(M)) - 1
        A_eq.append(a); b_eq.append(0)
    for d in range(D):  # y <= 1
        for q in range(Q):
            a = [0] * nv
            a[Y(d, q)] = 1
            A_ub.append(a); b_ub.append(1)
    for d in range(D):  # Eq. 4
        a = [0] * nv
        for q in range(Q):
            a[Z(d, q)] = 1
            a[Y(d, q)] = -int(demand[q])
        A_ub.append(a); b_ub.append(0)
    for d in range(D):  # Eq. 5
        for q in range(Q):
            a = [0] * nv
            a[Z(d, q)] = 1
            A_ub.append(a); b_ub.append(sum(Pdmq(d, m, q) * x[d][m] for m in range(M)))
    # stage 1 (C1): maximise total served
    c1 = [0] * nv
    for d in range(D):
        for q in range(Q):
            c1[Z(d, q)] = 1
    served, _ = lp_max(c1, A_ub, b_ub, A_eq, b_eq, presolve)
    # stage 2: Eq. 7 at the optimal served
    c2 = [0] * nv
    for d in range(D):
        for q in range(Q):
            c2[Z(d, q)] = sum(int(acc_m[m]) * x[d][m] for m in range(M))
    acc, sol = lp_max(c2, A_ub, b_ub, A_eq + [c1], b_eq + [served], presolve)
    z = [[sol[Z(d, q)] for q in range(Q)] for d in range(D)]
    return served, acc, z


def brute_force_fractional(P_tm, acc_m, V, device_type, option, demand, grid=2):
    """Toy-size check: every z_{d,q} on a 1/grid lattice within its bounds,
    keeping the feasible ones (Eqs. 2-6 with y = z / s); returns the
    lexicographic (served, accsum) maximum as Fractions."""
    V = list(map(int, V))
    Q = len(V)
    fam = [q for q in range(Q) for _ in range(V[q])]
    D = len(option)
    ranges = []
    for d in range(D):
        o = option[d]
        if o == 0:
            ranges.append([(None, Fr(0))])
            continue
        q = fam[o - 1]
        cap = int(P_tm[device_type[d]][o - 1])
        ranges.append([(q, Fr(k, grid)) for k in range(cap * grid + 1)])
    best = None
    idx = [0] * D
    while True:
        served_q = [Fr(0)] * Q
        acc = Fr(0)
        for d in range(D):
            q, zval = ranges[d][idx[d]]
            if q is not None:
                served_q[q] += zval
                acc += zval * int(acc_m[option[d] - 1])
        if all(served_q[q] <= int(demand[q]) for q in range(Q)):
            key = (sum(served_q), acc)
            if best is None or key > best:
                best = key
        k = D - 1
        while k >= 0:
            idx[k] += 1
            if idx[k] < len(ranges[k]):
                break
            idx[k] = 0
            k -= 1
        if k < 0:
            break
    return best


def np_int(x):
    return np.asarray(x, dtype=np.int64)
