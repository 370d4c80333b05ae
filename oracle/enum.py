"""O-8: brute-force enumeration of every fusion partition (the "deterministic method" the
paper uses to verify its search on small benchmarks).

Partitions of n kernels are listed as restricted-growth strings in lexicographic order
(Bell(n) of them); each is validated by oracle.legality.  The optimum minimises the total
compulsory bytes (Eq. 1 with the codeless projection T = bytes / BW); ties go to the
lexicographically smallest canonical labelling (reading R17).
"""
from __future__ import annotations

from typing import Iterator, List, Tuple

from workloads.program import Program

from . import legality as L


def restricted_growth(n: int) -> Iterator[List[int]]:
    if n == 0:
        yield []
        return
    a = [0] * n

    def rec(i, m):
        if i == n:
            yield list(a)
            return
        for v in range(m + 2):
            a[i] = v
            yield from rec(i + 1, max(m, v))
    a[0] = 0
    yield from rec(1, 0)


def bell(n: int) -> int:
    # Bell triangle
    row = [1]
    for _ in range(n - 1):
        nxt = [row[-1]]
        for x in row:
            nxt.append(nxt[-1] + x)
        row = nxt
    return row[-1] if n > 0 else 1


def legal_plans(prog: Program, target: L.Target = L.Target()) -> List[List[int]]:
    return [p for p in restricted_growth(len(prog.kernels)) if L.validate(prog, p, target)[0] == L.V_OK]


def best_plan(prog: Program, target: L.Target = L.Target()) -> Tuple[List[int], int]:
    best, best_b = None, None
    for p in restricted_growth(len(prog.kernels)):
        if L.validate(prog, p, target)[0] != L.V_OK:
            continue
        b = L.project(prog, p, target)[1]
        if best_b is None or b < best_b:
            best, best_b = p, b
    return best, best_b
