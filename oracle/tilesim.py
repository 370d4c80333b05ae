"""O-7: tile simulator -- executes a fused group the way a GPU thread block would.

Complex fusion as described at PAPER.md:107: each thread block computes the
producers of a group on "an extra layer(s) of stencil sites" (its extended
region) because on-chip memory is not coherent across blocks, and only
the sites "originally intended per thread block" are written back.

Per tile T (3D box), for each kernel of the group in program order, the kernel
is evaluated on the bounding box of its extended region E(k) (computed by
oracle.legality from point sets), clipped to the interior on FROZEN axes.
Inputs produced inside the group come from tile-local values; everything else
comes from the simulated HBM.  On frozen axes a read of an in-group value
outside the interior takes the stored ghost value (reading R9).  At the end of
the tile the live-out versions are stored on T ∩ interior.

Tile orders: "snapshot" (every tile reads before any tile writes) or any
permutation of sequential tiles.  A plan is hazard-free (V5) iff every order
reproduces oracle.interp bit for bit -- the semantic pin of V5 and of the
extended-region rule.  Relaxed arrays live in one buffer per version.
"""
from __future__ import annotations

import itertools
from typing import Dict, List, Optional, Sequence, Tuple

import numpy as np

from workloads.program import BC_PERIODIC, DT_F32, OP_LOAD, Program

from . import graph as G
from . import legality as L
from .interp import eval_rpn


class _Mem:
    """Simulated HBM: one ghosted buffer per array, plus one per version of relaxed arrays."""

    def __init__(self, prog: Program, inputs: Dict[str, np.ndarray]):
        self.prog = prog
        dt = np.float32 if prog.dtype == DT_F32 else np.float64
        self.buf: Dict[object, np.ndarray] = {}
        for x, (nm, _) in enumerate(prog.arrays):
            self.buf[x] = np.array(inputs[nm], dtype=dt, copy=True)

    def key(self, x: int, v: int):
        return (x, v) if (G.relaxed(self.prog, x) and v >= 1) else x

    def get(self, x: int, v: int) -> np.ndarray:
        k = self.key(x, v)
        if k not in self.buf:
            self.buf[k] = self.buf[x].copy()      # ghosts of a renamed copy = the array's ghosts
        return self.buf[k]

    def end_step(self):
        """Renamed final versions become the next step's version 0 (ping-pong / copy-back)."""
        prog = self.prog
        for x in range(len(prog.arrays)):
            if G.relaxed(prog, x):
                w = len(G.writers(prog, x))
                if w >= 1:
                    src = self.get(x, w)
                    self.buf[x][...] = src
                    for v in range(1, w + 1):
                        self.buf.pop((x, v), None)


def _region(prog: Program, tile_lo, tile_hi, ext) -> Optional[List[np.ndarray]]:
    """Coordinates of E(k) for this tile, clipped to the interior on frozen axes."""
    (lo, hi) = ext
    ax = []
    for a in range(3):
        s, e = tile_lo[a] - lo[a], tile_hi[a] + hi[a]      # [s, e)
        if prog.bc[a] != BC_PERIODIC:
            s, e = max(s, 0), min(e, prog.n[a])
        if e <= s:
            return None
        ax.append(np.arange(s, e))
    return ax


def refill_ghosts(prog: Program, mem: _Mem) -> None:
    """Ghost-limited mode: before a group, every buffer's ghost layer on PERIODIC axes is refreshed
    with the wrapped interior (what the device's ghost fills / ghost writes / halo exchanges
    provide), one axis after the other (x, then y over whole padded rows, then z planes)."""
    n, g = prog.n, prog.ghost
    for b in mem.buf.values():
        for a in range(3):
            if prog.bc[a] != BC_PERIODIC or g[a] == 0:
                continue
            ax = 2 - a
            lo = [slice(None)] * 3
            src = [slice(None)] * 3
            lo[ax], src[ax] = slice(0, g[a]), slice(n[a], n[a] + g[a])
            b[tuple(lo)] = b[tuple(src)]
            lo[ax], src[ax] = slice(g[a] + n[a], n[a] + 2 * g[a]), slice(g[a], 2 * g[a])
            b[tuple(lo)] = b[tuple(src)]


def run_group_tiles(prog: Program, grp: List[int], mem: _Mem, params, tile, order, ghost_limited=False) -> None:
    ext, _ = L.extended_regions(prog, grp)
    lout = L.live_out(prog, grp)
    n = prog.n
    g = prog.ghost
    ntiles = [-(-n[a] // tile[a]) for a in range(3)]
    tiles = list(itertools.product(range(ntiles[0]), range(ntiles[1]), range(ntiles[2])))
    pad = [max([0] + [max(abs(e[0][a]), abs(e[1][a])) for e in ext.values() if e is not None]) + tile[a] + 8
           for a in range(3)]
    dt = np.float32 if prog.dtype == DT_F32 else np.float64

    def wrapped(a, q):
        return q % n[a] if prog.bc[a] == BC_PERIODIC else q

    def hbm_load(x, v, qx, qy, qz):
        b = mem.get(x, v)
        if not ghost_limited:
            return b[np.ix_(wrapped(2, qz) + g[2], wrapped(1, qy) + g[1], wrapped(0, qx) + g[0])]
        # V6 pin: periodic neighbours only through the stored ghost layer of width ghost[a]; a read
        # beyond it has no defined value (NaN sentinel)
        idx, ok = [], []
        for a, q in ((2, qz), (1, qy), (0, qx)):
            i = q + g[a]
            ok.append((i >= 0) & (i < n[a] + 2 * g[a]))
            idx.append(np.clip(i, 0, n[a] + 2 * g[a] - 1))
        val = b[np.ix_(*idx)].copy()
        bad = ~(ok[0][:, None, None] & ok[1][None, :, None] & ok[2][None, None, :])
        val[bad] = np.nan
        return val

    def compute_tile(t):
        tlo = [t[a] * tile[a] for a in range(3)]
        thi = [min(tlo[a] + tile[a], n[a]) for a in range(3)]
        local: Dict[Tuple[int, int], np.ndarray] = {}
        for k in grp:
            if ext[k] is None:
                continue
            reg = _region(prog, tlo, thi, ext[k])
            if reg is None:
                continue
            rx, ry, rz = reg

            def get(x, d, k=k, rx=rx, ry=ry, rz=rz):
                v = G.version_read(prog, k, x)
                qx, qy, qz = rx + d[0], ry + d[1], rz + d[2]
                if v >= 1 and G.writer_of(prog, x, v) in grp:
                    loc = local.get((x, v))
                    if loc is None:
                        loc = np.full([n[2] + 2 * pad[2], n[1] + 2 * pad[1], n[0] + 2 * pad[0]], np.nan, dtype=dt)
                    val = loc[np.ix_(qz + pad[2], qy + pad[1], qx + pad[0])]
                    # frozen axes: outside the interior the stored ghost is read (R9)
                    out_mask = np.zeros(val.shape, dtype=bool)
                    for a, q in ((0, qx), (1, qy), (2, qz)):
                        if prog.bc[a] != BC_PERIODIC:
                            m = (q < 0) | (q >= n[a])
                            shape = [1, 1, 1]
                            shape[2 - a] = len(q)
                            out_mask |= m.reshape(shape)
                    if out_mask.any():
                        ghost = hbm_load(x, v, qx, qy, qz)
                        val = np.where(out_mask, ghost, val)
                    return val
                return hbm_load(x, v, qx, qy, qz)

            vals = [(s.out, eval_rpn(prog, s.rpn, get, params)) for s in prog.kernels[k].stmts]
            for out, val in vals:
                v = G.version_written(prog, k, out)
                arr = local.get((out, v))
                if arr is None:
                    arr = np.full([n[2] + 2 * pad[2], n[1] + 2 * pad[1], n[0] + 2 * pad[0]], np.nan, dtype=dt)
                    local[(out, v)] = arr
                arr[np.ix_(rz + pad[2], ry + pad[1], rx + pad[0])] = np.broadcast_to(val, (len(rz), len(ry), len(rx)))
        stores = []
        for (x, v) in lout:
            arr = local.get((x, v))
            if arr is None:
                continue
            sl = arr[pad[2] + tlo[2]:pad[2] + thi[2], pad[1] + tlo[1]:pad[1] + thi[1], pad[0] + tlo[0]:pad[0] + thi[0]]
            stores.append((x, v, tlo, thi, sl.copy()))
        return stores

    def commit(stores):
        for (x, v, tlo, thi, sl) in stores:
            b = mem.get(x, v)
            b[g[2] + tlo[2]:g[2] + thi[2], g[1] + tlo[1]:g[1] + thi[1], g[0] + tlo[0]:g[0] + thi[0]] = sl

    if order == "snapshot":
        all_st = [compute_tile(t) for t in tiles]
        for st in all_st:
            commit(st)
    else:
        for i in order:
            commit(compute_tile(tiles[i]))


def n_tiles(prog: Program, tile) -> int:
    return int(np.prod([-(-prog.n[a] // tile[a]) for a in range(3)]))


def run_fused(prog: Program, plan: List[int], inputs: Dict[str, np.ndarray], nsteps: int, tile,
              order="snapshot", params=None, ghost_limited=False) -> Dict[str, np.ndarray]:
    """Run `nsteps` of the fused plan (groups in quotient-topological order, R18).  ghost_limited:
    periodic reads go through ghost layers of the declared width, refreshed before every group
    (the semantic pin of V6's ghost rule)."""
    params = list(prog.params if params is None else params)
    mem = _Mem(prog, inputs)
    gs = L.groups_of(plan)
    qo = L.quotient_order(prog, plan)
    assert qo is not None, "plan has a cyclic quotient graph"
    with np.errstate(all="ignore"):
        for _ in range(nsteps):
            for g in qo:
                if ghost_limited:
                    refill_ghosts(prog, mem)
                run_group_tiles(prog, gs[g], mem, params, tile, order, ghost_limited)
            mem.end_step()
    return {nm: mem.buf[i] for i, (nm, _) in enumerate(prog.arrays)}
