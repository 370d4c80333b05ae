"""Program description shared by the oracle and the CUDA path (input only).

This module holds NO arithmetic of the method: it only describes a stencil
program -- the paper's input "original kernels K, |K| = n; data arrays D,
|D| = l" (Fig. 4) -- as plain data, plus a tiny expression DSL
that writes kernel bodies as RPN.  Both `oracle/` and the C-ABI binding read
this description; neither depends on the other.

Encoding (mirrors include/kf.h `kf_insn`):
  op    one of the OP_* codes below
  arg   LOAD: array index, PARAM: parameter index
  d     LOAD: (di, dj, dk) offset, x fastest
  imm   CONST: value (rounded to the program dtype by whoever evaluates it)
RPN is evaluated left to right, one IEEE operation per node.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Dict, List, Optional, Sequence, Tuple

OP_CONST, OP_PARAM, OP_LOAD, OP_ADD, OP_SUB, OP_MUL, OP_DIV, OP_MIN, OP_MAX, OP_NEG, OP_ABS, OP_SQRT = range(12)
OP_NAMES = ["CONST", "PARAM", "LOAD", "ADD", "SUB", "MUL", "DIV", "MIN", "MAX", "NEG", "ABS", "SQRT"]
BINARY = {OP_ADD, OP_SUB, OP_MUL, OP_DIV, OP_MIN, OP_MAX}
UNARY = {OP_NEG, OP_ABS, OP_SQRT}

ARRAY_OUTPUT = 1 << 0
ARRAY_READONLY = 1 << 1

PROG_RELAX_EXPANDABLE = 1 << 0   # paper P:53: rename expandable arrays
PROG_RELAX_ALL = 1 << 1          # extension: rename every written array
PROG_NO_KINSHIP = 1 << 2         # experiments only: skip constraint (1.5)

BC_FROZEN, BC_PERIODIC = 0, 1
DT_F32, DT_F64 = 0, 1


@dataclass(frozen=True)
class Insn:
    op: int
    arg: int = 0
    d: Tuple[int, int, int] = (0, 0, 0)
    imm: float = 0.0


@dataclass
class Stmt:
    out: int                 # array index written
    rpn: List[Insn]


@dataclass
class Kernel:
    name: str
    stmts: List[Stmt]

    def reads(self) -> Dict[int, List[Tuple[int, int, int]]]:
        """array -> sorted distinct LOAD offsets (the kernel's stencil footprint)."""
        r: Dict[int, set] = {}
        for s in self.stmts:
            for ins in s.rpn:
                if ins.op == OP_LOAD:
                    r.setdefault(ins.arg, set()).add(tuple(ins.d))
        return {a: sorted(v) for a, v in sorted(r.items())}

    def writes(self) -> List[int]:
        return [s.out for s in self.stmts]


@dataclass
class Program:
    name: str
    dtype: int                              # DT_F32 / DT_F64
    n: Tuple[int, int, int]                 # interior extents (nx, ny, nz)
    ghost: Tuple[int, int, int]
    bc: Tuple[int, int, int]                # BC_FROZEN / BC_PERIODIC per axis
    arrays: List[Tuple[str, int]]           # (name, flags)
    kernels: List[Kernel]
    params: List[float] = field(default_factory=list)   # default values of PARAM slots
    flags: int = 0

    @property
    def es(self) -> int:
        return 4 if self.dtype == DT_F32 else 8

    @property
    def npts(self) -> int:
        return self.n[0] * self.n[1] * self.n[2]

    def array_index(self, name: str) -> int:
        for i, (nm, _) in enumerate(self.arrays):
            if nm == name:
                return i
        raise KeyError(name)

    def padded_shape(self) -> Tuple[int, int, int]:
        """Logical ghosted shape (z, y, x) used by generators and the oracle."""
        nx, ny, nz = self.n
        gx, gy, gz = self.ghost
        return (nz + 2 * gz, ny + 2 * gy, nx + 2 * gx)

    def with_(self, **kw) -> "Program":
        d = dict(self.__dict__)
        d.update(kw)
        return Program(**d)


# --------------------------------------------------------------------------
# expression DSL -> RPN (left-to-right post-order; one node = one IEEE op)
# --------------------------------------------------------------------------
class E:
    __slots__ = ("op", "arg", "d", "imm", "kids")

    def __init__(self, op, arg=0, d=(0, 0, 0), imm=0.0, kids=()):
        self.op, self.arg, self.d, self.imm, self.kids = op, arg, tuple(d), float(imm), tuple(kids)

    @staticmethod
    def lift(x) -> "E":
        if isinstance(x, E):
            return x
        return E(OP_CONST, imm=float(x))

    def _bin(self, op, o, rev=False):
        o = E.lift(o)
        return E(op, kids=(o, self) if rev else (self, o))

    def __add__(self, o): return self._bin(OP_ADD, o)
    def __radd__(self, o): return self._bin(OP_ADD, o, True)
    def __sub__(self, o): return self._bin(OP_SUB, o)
    def __rsub__(self, o): return self._bin(OP_SUB, o, True)
    def __mul__(self, o): return self._bin(OP_MUL, o)
    def __rmul__(self, o): return self._bin(OP_MUL, o, True)
    def __truediv__(self, o): return self._bin(OP_DIV, o)
    def __rtruediv__(self, o): return self._bin(OP_DIV, o, True)
    def __neg__(self): return E(OP_NEG, kids=(self,))


def emin(a, b) -> E: return E(OP_MIN, kids=(E.lift(a), E.lift(b)))
def emax(a, b) -> E: return E(OP_MAX, kids=(E.lift(a), E.lift(b)))
def eabs(a) -> E: return E(OP_ABS, kids=(E.lift(a),))
def esqrt(a) -> E: return E(OP_SQRT, kids=(E.lift(a),))


def to_rpn(e: E) -> List[Insn]:
    out: List[Insn] = []

    def rec(x: E):
        for k in x.kids:
            rec(k)
        out.append(Insn(x.op, x.arg, x.d, x.imm))
    rec(E.lift(e))
    return out


class ArrayRef:
    """Handle returned by Builder.array; A[di,dj,dk] (or A with no index) loads."""

    def __init__(self, idx: int, name: str):
        self.idx, self.name = idx, name

    def __getitem__(self, d) -> E:
        if not isinstance(d, tuple):
            d = (d,)
        d = tuple(d) + (0,) * (3 - len(d))
        return E(OP_LOAD, arg=self.idx, d=d)

    @property
    def c(self) -> E:
        return self[0, 0, 0]


class Builder:
    def __init__(self, name, dtype, n, ghost, bc, flags=0):
        self.name, self.dtype, self.n, self.ghost, self.bc, self.flags = name, dtype, tuple(n), tuple(ghost), tuple(bc), flags
        self.arrays: List[Tuple[str, int]] = []
        self.kernels: List[Kernel] = []
        self.params: List[float] = []
        self._refs: Dict[str, ArrayRef] = {}

    def array(self, name: str, flags: int = 0) -> ArrayRef:
        r = ArrayRef(len(self.arrays), name)
        self.arrays.append((name, flags))
        self._refs[name] = r
        return r

    def param(self, value: float) -> E:
        self.params.append(float(value))
        return E(OP_PARAM, arg=len(self.params) - 1)

    def kernel(self, name: str, *stmts: Tuple[ArrayRef, E]):
        self.kernels.append(Kernel(name, [Stmt(a.idx, to_rpn(e)) for a, e in stmts]))

    def build(self) -> Program:
        return Program(self.name, self.dtype, self.n, self.ghost, self.bc, list(self.arrays),
                       list(self.kernels), list(self.params), self.flags)


def footprint_radius(prog: Program) -> Tuple[int, int, int]:
    """Largest |offset| per axis over all LOADs (single-kernel radius)."""
    r = [0, 0, 0]
    for k in prog.kernels:
        for offs in k.reads().values():
            for d in offs:
                for a in range(3):
                    r[a] = max(r[a], abs(d[a]))
    return tuple(r)


def unroll(prog: Program, steps: int) -> Program:
    """Temporal unrolling (NEXT-4, the temporal blocking of [15] cited at P:107 / P:556): the
    description of `steps` consecutive timesteps as ONE step -- the kernel list repeated `steps`
    times in order over the same arrays (kernel names suffixed with the sub-step).  Running the
    result for N steps is, by definition, running `prog` for N*steps steps; a fusion plan of it may
    group kernels of consecutive timesteps.  Pure description (no arithmetic of the method)."""
    assert steps >= 1
    kernels = [Kernel(f"{k.name}@{s}", [Stmt(st.out, list(st.rpn)) for st in k.stmts])
               for s in range(steps) for k in prog.kernels]
    return prog.with_(name=prog.name if steps == 1 else f"{prog.name}x{steps}", kernels=kernels)


def disjoint_union(parts: Sequence[Program], seed: int = 0) -> Tuple[Program, List[int]]:
    """One program made of independent sub-programs: the arrays of every part renamed apart
    (part index prefix), the kernels interleaved in a seeded random order that keeps each part's
    own kernel order.  Returns the program and, per kernel, the part it came from.  Parts share
    no array, so no dependence, sharing set or kinship chain crosses two parts: a legal group lies
    inside one part and a plan of the union is a plan per part (the search pin at 40+ kernels).
    All parts must have the same dtype, grid, ghost, boundary conditions and flags; PARAM slots
    are re-indexed.  Pure description (no arithmetic of the method)."""
    import numpy as np
    p0 = parts[0]
    for q in parts[1:]:
        assert (q.dtype, tuple(q.n), tuple(q.ghost), tuple(q.bc), q.flags) == \
            (p0.dtype, tuple(p0.n), tuple(p0.ghost), tuple(p0.bc), p0.flags)
    arrays, params, aoff, poff = [], [], [], []
    for i, q in enumerate(parts):
        aoff.append(len(arrays))
        poff.append(len(params))
        arrays += [(f"p{i}_{nm}", fl) for nm, fl in q.arrays]
        params += list(q.params)
    queues = [list(range(len(q.kernels))) for q in parts]
    order = [i for i, q in enumerate(parts) for _ in q.kernels]
    np.random.default_rng(seed).shuffle(order)
    kernels, part_of = [], []
    for i in order:
        k = parts[i].kernels[queues[i].pop(0)]

        def mv(ins: Insn, i=i) -> Insn:
            if ins.op == OP_LOAD:
                return Insn(ins.op, ins.arg + aoff[i], ins.d, ins.imm)
            if ins.op == OP_PARAM:
                return Insn(ins.op, ins.arg + poff[i], ins.d, ins.imm)
            return ins
        kernels.append(Kernel(f"p{i}_{k.name}", [Stmt(st.out + aoff[i], [mv(x) for x in st.rpn]) for st in k.stmts]))
        part_of.append(i)
    return p0.with_(name="union_" + "_".join(q.name for q in parts), arrays=arrays, kernels=kernels,
                    params=params), part_of
