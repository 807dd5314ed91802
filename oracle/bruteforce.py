"""Brute-force optimal placement on tiny job sets (pins for the balancer).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Objective (SURVEY.md §8(c) "DTF/MBF placement"): the static vector load
    L(pi) = max_d max_k  sum_{j : pi(j) = d} p_jk
over resources k (each job j has a load vector p_j).  Enumerates all G^J
placements, so only for J <= 8, G <= 3.
"""
from __future__ import annotations

import itertools
from typing import List, Sequence, Tuple


def vector_load(loads: Sequence[Sequence[int]], placement: Sequence[int], G: int) -> int:
    K = len(loads[0]) if loads else 0
    acc = [[0] * K for _ in range(G)]
    for j, d in enumerate(placement):
        for k in range(K):
            acc[d][k] += loads[j][k]
    return max((max(row) if row else 0) for row in acc)


def optimal_vector_load(loads: Sequence[Sequence[int]], G: int) -> Tuple[int, Tuple[int, ...]]:
    assert len(loads) <= 8 and G <= 3, "brute force only for tiny cases"
    best, arg = None, None
    for pl in itertools.product(range(G), repeat=len(loads)):
        v = vector_load(loads, pl, G)
        if best is None or v < best:
            best, arg = v, pl
    return best, arg
