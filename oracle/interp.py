"""O-1: semantics interpreter -- the unfused program, kernel by kernel, in program order.

Follows the paper's original kernels: every thread owns one (i, j) column and
loops over k (Listings 1-5); "each CUDA thread loads a single
stencil site".  Kernels run in their original order (the order of
execution must not be violated).  Readings:
  R1  all reads of a kernel see pre-kernel values (statements are evaluated,
      then committed); a kernel may read an array it writes only at offset 0.
  R9  per-axis boundary: FROZEN reads the stored ghost cell (never written),
      PERIODIC wraps modulo n.
  R16 every RPN node is one IEEE op in the program dtype, left to right;
      CONST / PARAM rounded to the dtype; MIN(a,b) := (b<a)?b:a,
      MAX(a,b) := (a<b)?b:a; no FMA contraction (numpy never contracts).
Vectorised over the whole interior: each op is elementwise, so this equals
scalar evaluation point by point.
"""
from __future__ import annotations

from typing import Dict, Optional, Sequence

import numpy as np

from workloads.program import (BC_PERIODIC, DT_F32, OP_ABS, OP_ADD, OP_CONST, OP_DIV, OP_LOAD,
                               OP_MAX, OP_MIN, OP_MUL, OP_NEG, OP_PARAM, OP_SQRT, OP_SUB, Program)


def _dt(prog: Program):
    return np.float32 if prog.dtype == DT_F32 else np.float64


def _axis_index(prog: Program, axis: int, d: int) -> np.ndarray:
    """Ghosted-array indices of the interior points shifted by d along `axis` (R9)."""
    n, g = prog.n[axis], prog.ghost[axis]
    idx = np.arange(n) + d
    if prog.bc[axis] == BC_PERIODIC:
        idx = idx % n
    else:
        assert np.all(idx >= -g) and np.all(idx < n + g), "read beyond the ghost layer"
    return idx + g


def load(prog: Program, arr: np.ndarray, d: Sequence[int]) -> np.ndarray:
    ix = _axis_index(prog, 0, d[0])
    iy = _axis_index(prog, 1, d[1])
    iz = _axis_index(prog, 2, d[2])
    return arr[np.ix_(iz, iy, ix)]


def eval_rpn(prog: Program, rpn, get, params) -> np.ndarray:
    """Evaluate one statement.  `get(array, d)` returns the loaded operand."""
    dt = _dt(prog)
    st = []
    for ins in rpn:
        op = ins.op
        if op == OP_CONST:
            st.append(dt(ins.imm))
        elif op == OP_PARAM:
            st.append(dt(params[ins.arg]))
        elif op == OP_LOAD:
            st.append(get(ins.arg, ins.d))
        elif op in (OP_NEG, OP_ABS, OP_SQRT):
            a = st.pop()
            st.append(-a if op == OP_NEG else (np.abs(a) if op == OP_ABS else np.sqrt(a)))
        else:
            b = st.pop()
            a = st.pop()
            if op == OP_ADD:
                r = a + b
            elif op == OP_SUB:
                r = a - b
            elif op == OP_MUL:
                r = a * b
            elif op == OP_DIV:
                r = a / b
            elif op == OP_MIN:
                r = np.where(b < a, b, a)
            elif op == OP_MAX:
                r = np.where(a < b, b, a)
            else:
                raise ValueError(op)
            st.append(np.asarray(r, dtype=dt) if np.ndim(r) == 0 else r.astype(dt, copy=False))
    assert len(st) == 1
    return st[0]


def run_kernel(prog: Program, k: int, arrs, params) -> None:
    """One original kernel over the whole interior: evaluate all statements, then commit (R1)."""
    kern = prog.kernels[k]
    nx, ny, nz = prog.n
    gx, gy, gz = prog.ghost
    vals = []
    for s in kern.stmts:
        v = eval_rpn(prog, s.rpn, lambda a, d: load(prog, arrs[a], d), params)
        vals.append((s.out, np.broadcast_to(v, (nz, ny, nx))))
    for out, v in vals:
        arrs[out][gz:gz + nz, gy:gy + ny, gx:gx + nx] = v


def run(prog: Program, inputs: Dict[str, np.ndarray], nsteps: int,
        params: Optional[Sequence[float]] = None, kernels: Optional[Sequence[int]] = None) -> Dict[str, np.ndarray]:
    """Run `nsteps` steps of the unfused program; returns new arrays (inputs untouched)."""
    params = list(prog.params if params is None else params)
    arrs = [np.array(inputs[nm], dtype=_dt(prog), copy=True) for nm, _ in prog.arrays]
    ks = range(len(prog.kernels)) if kernels is None else kernels
    with np.errstate(all="ignore"):
        for _ in range(nsteps):
            for k in ks:
                run_kernel(prog, k, arrs, params)
    return {nm: arrs[i] for i, (nm, _) in enumerate(prog.arrays)}
