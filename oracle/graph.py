"""O-2/O-3/O-4: versions, precedence DAG, array classes, sharing sets, kinship, liveness.

Plain definitions, written from PAPER.md §II-D.1-2 and Table II:
  * data-dependency graph: kernels and arrays, read and write edges
  * array classes read-only / read-write / expandable read-write / write-only
  * order-of-execution graph: the inter-kernel precedences "extracted from data
    dependencies", relaxed for expandable arrays by redundant arrays
  * sharing set K(D), degree of kinship (Table II)
Readings R2 (which precedences), R3 (path closure on the full DAG), R5 (kinship
chain inside the group), R15 (liveness) -- see DESIGN.md.
"""
from __future__ import annotations

from typing import Dict, List, Set, Tuple

from workloads.program import ARRAY_OUTPUT, PROG_RELAX_ALL, PROG_RELAX_EXPANDABLE, Program

RAW, WAR, WAW = 0, 1, 2
CLS_RO, CLS_RW, CLS_EXPANDABLE, CLS_WO = 0, 1, 2, 3


def reads(prog: Program, k: int) -> Dict[int, List[Tuple[int, int, int]]]:
    return prog.kernels[k].reads()


def writes(prog: Program, k: int) -> List[int]:
    return prog.kernels[k].writes()


def writers(prog: Program, x: int) -> List[int]:
    return [k for k in range(len(prog.kernels)) if x in writes(prog, k)]


def readers_of_array(prog: Program, x: int) -> List[int]:
    return [k for k in range(len(prog.kernels)) if x in reads(prog, k)]


def version_read(prog: Program, k: int, x: int) -> int:
    """Version of x current just before kernel k = number of earlier kernels writing x."""
    return sum(1 for j in range(k) if x in writes(prog, j))


def version_written(prog: Program, k: int, x: int) -> int:
    return version_read(prog, k, x) + 1


def writer_of(prog: Program, x: int, v: int) -> int:
    """Kernel producing version v >= 1 of x."""
    return writers(prog, x)[v - 1]


def readers_of_version(prog: Program, x: int, v: int) -> List[int]:
    return [k for k in readers_of_array(prog, x) if version_read(prog, k, x) == v]


def array_class(prog: Program, x: int) -> int:
    """P:49-54.  RO: never written.  WO: written, never read.  EXPANDABLE: >= 2 writers."""
    nw, nr = len(writers(prog, x)), len(readers_of_array(prog, x))
    if nw == 0:
        return CLS_RO
    if nr == 0:
        return CLS_WO
    if nw >= 2:
        return CLS_EXPANDABLE
    return CLS_RW


def relaxed(prog: Program, x: int) -> bool:
    """Arrays renamed by redundant copies (P:53 'writing into redundant arrays')."""
    if prog.flags & PROG_RELAX_ALL:
        return len(writers(prog, x)) >= 1
    if prog.flags & PROG_RELAX_EXPANDABLE:
        return array_class(prog, x) == CLS_EXPANDABLE
    return False


def edges(prog: Program) -> List[Tuple[int, int, int, int]]:
    """Canonical precedence edges (src, dst, kind, array), sorted by (dst, src, kind, array).

    RAW from the writer of the version read; for arrays that are not relaxed also WAW from
    the previous writer and WAR from every reader of the overwritten version (reading R2)."""
    out = set()
    nk = len(prog.kernels)
    for b in range(nk):
        for x in reads(prog, b):
            v = version_read(prog, b, x)
            if v >= 1:
                out.add((writer_of(prog, x, v), b, RAW, x))
        for x in writes(prog, b):
            if relaxed(prog, x):
                continue
            v = version_read(prog, b, x)
            if v >= 1:
                out.add((writer_of(prog, x, v), b, WAW, x))
            for a in readers_of_version(prog, x, v):
                if a < b:
                    out.add((a, b, WAR, x))
    return sorted(out, key=lambda e: (e[1], e[0], e[2], e[3]))


def all_pairs_hazards(prog: Program) -> Set[Tuple[int, int]]:
    """Every pair a<b with a RAW/WAR/WAW on a shared array (the un-canonicalised definition,
    relaxation applied per array as in `edges`) -- used to cross-check the closure."""
    out = set()
    nk = len(prog.kernels)
    for a in range(nk):
        Ra, Wa = set(reads(prog, a)), set(writes(prog, a))
        for b in range(a + 1, nk):
            Rb, Wb = set(reads(prog, b)), set(writes(prog, b))
            for x in (Wa & Rb):
                # RAW only if b reads the version a wrote or a later one derived through writers
                if not relaxed(prog, x) or version_read(prog, b, x) == version_written(prog, a, x):
                    out.add((a, b))
            for x in (Ra & Wb) | (Wa & Wb):
                if not relaxed(prog, x):
                    out.add((a, b))
    return out


def closure(n: int, es) -> List[List[bool]]:
    """reach[a][b]: a path of length >= 1 from a to b (Floyd-Warshall)."""
    r = [[False] * n for _ in range(n)]
    for e in es:
        r[e[0]][e[1]] = True
    for k in range(n):
        for i in range(n):
            if r[i][k]:
                for j in range(n):
                    if r[k][j]:
                        r[i][j] = True
    return r


def touched(prog: Program, k: int) -> Set[int]:
    return set(reads(prog, k)) | set(writes(prog, k))


def sharing_set(prog: Program, x: int) -> List[int]:
    """K(D): kernels sharing use of array D (Table II)."""
    return [k for k in range(len(prog.kernels)) if x in touched(prog, k)]


def shares(prog: Program, a: int, b: int) -> bool:
    return a != b and bool(touched(prog, a) & touched(prog, b))


def kinship(prog: Program, a: int, b: int, group: List[int]) -> int:
    """(a,b)deg: length of the shortest chain of kernels inside `group`, consecutive ones
    sharing an array; 0 if none (Table II; reading R5)."""
    if a == b:
        return 0
    dist = {a: 0}
    frontier = [a]
    while frontier:
        nxt = []
        for u in frontier:
            for w in group:
                if w not in dist and shares(prog, u, w):
                    dist[w] = dist[u] + 1
                    nxt.append(w)
        frontier = nxt
    return dist.get(b, 0)


def step_live(prog: Program, x: int) -> bool:
    """A written array whose final value must reach HBM at the end of a step (R15):
    upward-exposed read, OUTPUT flag, or a final version nobody reads."""
    ws = writers(prog, x)
    if not ws:
        return False
    if readers_of_version(prog, x, 0):
        return True
    if prog.arrays[x][1] & ARRAY_OUTPUT:
        return True
    return len(readers_of_version(prog, x, len(ws))) == 0


def pivot(prog: Program, group: List[int]) -> Set[int]:
    """F^Pivot: arrays touched by >= 2 kernels of the group (reused on chip; Table II)."""
    return {x for x in range(len(prog.arrays)) if sum(1 for k in group if x in touched(prog, k)) >= 2}
