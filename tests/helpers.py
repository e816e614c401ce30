"""Comparison helpers shared by the test files (no method arithmetic here)."""
from __future__ import annotations

import os

import numpy as np

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")

# |c - c_ref| <= REL_TOL * sum|a_ik * b_kj|  per entry (BASELINE.json north_star)
REL_TOL = 1e-12


def read_golden_kv(name: str) -> dict:
    out = {}
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            k, v = line.split()
            out[k] = int(v)
    return out


def read_golden_matrix(name: str) -> np.ndarray:
    rows = []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                rows.append([float(x) for x in line.split()])
    return np.array(rows)


def values_close(got: np.ndarray, ref: np.ndarray, absref: np.ndarray, rel: float = REL_TOL) -> np.ndarray:
    """Element-wise acceptance: NaN matches NaN, +-Inf match exactly, else |d| <= rel*absref."""
    got = np.asarray(got, dtype=np.float64)
    ref = np.asarray(ref, dtype=np.float64)
    both_nan = np.isnan(got) & np.isnan(ref)
    inf = np.isinf(ref) | np.isinf(got)
    same_inf = inf & (got == ref)
    with np.errstate(invalid="ignore"):
        ok = np.abs(got - ref) <= rel * np.asarray(absref, dtype=np.float64)
    return both_nan | same_inf | (ok & ~inf)


def assert_values_close(got, ref, absref, rel: float = REL_TOL, what: str = "values"):
    ok = values_close(got, ref, absref, rel)
    if not ok.all():
        bad = np.flatnonzero(~ok)[:5]
        raise AssertionError(f"{what}: {np.count_nonzero(~ok)} entries out of tolerance, e.g. "
                             f"{[(int(i), float(got[i]), float(ref[i]), float(absref[i])) for i in bad]}")


def bitwise_equal_values(got, ref) -> bool:
    """Bitwise equality treating +0 == -0 and NaN == NaN."""
    got = np.asarray(got, dtype=np.float64)
    ref = np.asarray(ref, dtype=np.float64)
    if got.shape != ref.shape:
        return False
    nan = np.isnan(got) & np.isnan(ref)
    return bool(np.all((got == ref) | nan))


def csr_dense(m, n, rowptr, col, val) -> np.ndarray:
    D = np.zeros((m, n))
    rows = np.repeat(np.arange(m), np.diff(rowptr))
    D[rows, col] = val
    return D


def csr_pattern(m, n, rowptr, col) -> np.ndarray:
    P = np.zeros((m, n), dtype=bool)
    rows = np.repeat(np.arange(m), np.diff(rowptr))
    P[rows, col] = True
    return P
