#!/usr/bin/env python
"""Regenerate the C1 tile statistics of tests/golden/c1_poisson2d64.txt with scipy only.

The numbers were first measured during the survey with throwaway scripts; this
is the committed, independent provenance: it builds the 5-point Laplacian of a 64x64 grid with
scipy.sparse (x fastest), squares it with scipy, and counts the paper's tile-level quantities
from the sparsity patterns directly -- no code from oracle/ or from the CUDA path:

* tiles_a          non-empty 16x16 tiles of A (Section 3.2)
* tiles_structural |C'| with C' = A'B' over the tile patterns (the paper's step 1)
* tiles_c          non-empty tiles of C = A^2 (the exported C stores no empty tile, reading A6)
* pairs_structural tile pairs (A_IK, B_KJ) with both tiles stored
* pairs            the pairs that carry a product: colOcc(A_IK) & rowOcc(B_KJ) != 0 (reading B3)
* nnz_a, nnz_c, products  (products = sum_i sum_{k in A(i,:)} nnz(A(k,:)), Table 2)

    python scripts/golden_c1_stats.py            # print the key/value lines
    python scripts/golden_c1_stats.py --check    # compare with tests/golden/c1_poisson2d64.txt
"""
from __future__ import annotations

import os
import sys

import numpy as np
import scipy.sparse as sp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
T = 16


def poisson2d(g: int) -> sp.csr_matrix:
    """5-point Laplacian on a g x g grid, x fastest (values irrelevant for the counts)."""
    one = sp.identity(g, format="csr")
    tri = sp.diags([np.ones(g - 1), 2 * np.ones(g), np.ones(g - 1)], [-1, 0, 1], format="csr")
    A = (sp.kron(one, tri) + sp.kron(tri, one)).tocsr()
    A.data[:] = 1.0
    return A


def tile_pattern(M: sp.csr_matrix) -> sp.csr_matrix:
    """Boolean (tm x tn) matrix of the non-empty 16x16 tiles."""
    C = M.tocoo()
    tm, tn = -(-M.shape[0] // T), -(-M.shape[1] // T)
    P = sp.coo_matrix((np.ones(C.nnz), (C.row // T, C.col // T)), shape=(tm, tn)).tocsr()
    P.data[:] = 1.0
    return P


def stats(A: sp.csr_matrix) -> dict:
    A = A.tocsr()
    A.sum_duplicates()
    Ab = A.copy()
    Ab.data[:] = 1.0
    C = (Ab @ Ab).tocsr()
    rownnz = np.diff(Ab.indptr)
    products = int(rownnz[Ab.indices].sum())
    PA = tile_pattern(Ab)
    Cp = (PA @ PA).tocsr()  # C' = A'B' (B = A)
    pairs_structural = int(Cp.sum())
    # contributing pairs: for tiles (I,K) of A and (K,J) of A, some (r, c) in A_IK with row c of
    # A_KJ non-empty; count them per (I, K, J) from the element-level pattern
    coo = Ab.tocoo()
    tr, tc = coo.row // T, coo.col // T
    pairs = 0
    occ = {}  # (K, J) -> set of local rows c of tile (K, J) that are non-empty
    for r, c in zip(coo.row, coo.col):
        occ.setdefault((r // T, c // T), set()).add(r % T)
    colocc = {}  # (I, K) -> set of local columns c of tile (I, K) that are non-empty
    for r, c in zip(coo.row, coo.col):
        colocc.setdefault((r // T, c // T), set()).add(c % T)
    by_row = {}
    for (K, J), rows in occ.items():
        by_row.setdefault(K, []).append((J, rows))
    for (I, K), cols in colocc.items():
        for J, rows in by_row.get(K, []):
            if cols & rows:
                pairs += 1
    return {"nnz_a": int(Ab.nnz), "nnz_c": int(C.nnz), "products": products, "tiles_a": int(PA.nnz),
            "tiles_structural": int(Cp.nnz), "tiles_c": int(tile_pattern(C).nnz),
            "pairs_structural": pairs_structural, "pairs": pairs}


def main() -> int:
    got = stats(poisson2d(64))
    if "--check" in sys.argv:
        gold = {}
        for ln in open(os.path.join(ROOT, "tests", "golden", "c1_poisson2d64.txt")):
            ln = ln.strip()
            if ln and not ln.startswith("#"):
                k, v = ln.split()
                gold[k] = int(v)
        bad = {k: (gold[k], got.get(k)) for k in gold if gold[k] != got.get(k)}
        print("golden matches scipy" if not bad else f"MISMATCH {bad}")
        return 1 if bad else 0
    for k, v in got.items():
        print(k, v)
    return 0


if __name__ == "__main__":
    sys.exit(main())
