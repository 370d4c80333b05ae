"""O-5/O-6/O-9: legality of a fusion plan, compulsory bytes, codeless projection.

Plain definitions from PAPER.md §III-B (Fig. 4, Eq. 1-1.7) and
§II-D (simple/complex fusion, halo layers), with readings R3-R8 of
DESIGN.md.  Checks run in the canonical order V1..V8; the first violation wins
(group-major inside each check).  Extended regions are computed by explicit
point-set propagation on a small tile and read back as bounding boxes -- the
library computes them with per-axis interval arithmetic instead.

V1 PARTITION  each kernel in exactly one new kernel (1.2, 1.4)
V2 KINSHIP    every pair in a group has degree of kinship > 0 (1.5)
V3 CONVEX     path closure: kernels on a path between two fused kernels are fused too (1.3)
V4 CYCLE      the groups can be ordered (quotient graph acyclic; reading R4)
V5 HAZARD     no cross-tile read of an array the group overwrites in HBM
              (SMEM incoherence across blocks; reading R7)
V6 HALO       accumulated halo fits the ghost layer on periodic/internal axes and max_halo
V7 SMEM       on-chip bytes <= capacity (1.6)    -- resource model, a definition (R20)
V8 REGS       registers <= R_Max (1.7)           -- resource model, a definition (R20)
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Dict, List, Optional, Tuple

from workloads.program import BC_PERIODIC, OP_ABS, OP_LOAD, OP_NEG, OP_SQRT, OP_CONST, OP_PARAM, Program

from . import graph as G

V_OK, V1_PARTITION, V2_KINSHIP, V3_CONVEX, V4_CYCLE, V5_HAZARD, V6_HALO, V7_SMEM, V8_REGS = range(9)


@dataclass
class Target:
    """Table IV analogue for B200."""
    hbm_bytes_per_s: float = 8.0e12
    smem_per_block: int = 232448
    regs_per_thread_max: int = 255
    n_sm: int = 148
    tile: Tuple[int, int, int] = (64, 4, 0)
    stages: int = 2
    threads: int = 256
    max_halo: int = 16
    internal_axes: int = 0          # bitmask of axes split across ranks (treated like periodic by V6)
    zunroll: int = 1                # planes per stream iteration U (ring depth grows with U, R20)
    pblock: Tuple[int, int] = (1, 1)  # points per thread in x, y (register blocking)
    ringunroll: int = 0             # 1: ring depths rounded up to powers of two (R20b)
    skew: int = 0                   # 1: reads at a nonzero xy offset of in-group versions lag U more planes (R20c)


# ---------------------------------------------------------------- plans
def canonical(plan: List[int]) -> List[int]:
    """Relabel groups in order of first appearance (restricted-growth string)."""
    m: Dict[int, int] = {}
    out = []
    for p in plan:
        if p not in m:
            m[p] = len(m)
        out.append(m[p])
    return out


def groups_of(plan: List[int]) -> List[List[int]]:
    c = canonical(plan)
    gs: List[List[int]] = [[] for _ in range(max(c) + 1)] if c else []
    for k, g in enumerate(c):
        gs[g].append(k)
    return gs


def live_in(prog: Program, grp: List[int]) -> List[Tuple[int, int]]:
    """Versions read by the group and not produced inside it (sorted (array, version))."""
    s = set()
    for k in grp:
        for x in G.reads(prog, k):
            v = G.version_read(prog, k, x)
            if v == 0 or G.writer_of(prog, x, v) not in grp:
                s.add((x, v))
    return sorted(s)


def live_out(prog: Program, grp: List[int]) -> List[Tuple[int, int]]:
    """Versions produced in the group that must reach HBM (R15): read by a kernel outside the
    group, or the final version of a step-live array."""
    s = set()
    for k in grp:
        for x in G.writes(prog, k):
            v = G.version_written(prog, k, x)
            rd = G.readers_of_version(prog, x, v)
            final = v == len(G.writers(prog, x))
            if any(r not in grp for r in rd) or (final and G.step_live(prog, x)):
                s.add((x, v))
    return sorted(s)


# ---------------------------------------------------------------- extended regions (point sets)
PT = (3, 3, 3)   # tile used for point-set propagation; bounding-box extents do not depend on it


def extended_regions(prog: Program, grp: List[int]):
    """E(k) for every k in the group, by explicit point sets (reading R8 / P:107 halo layers):
       E(k) = [T if k writes a live-out version] U  U_{c in G reads a version k wrote} E(c) (+) F_c(x)
    Returns {k: (lo[3], hi[3])} extents beyond T (may be negative), or None for an empty region."""
    T = {(x, y, z) for x in range(PT[0]) for y in range(PT[1]) for z in range(PT[2])}
    lo = set(live_out(prog, grp))
    pts: Dict[int, set] = {}
    for k in sorted(grp, reverse=True):
        s = set()
        if any((x, G.version_written(prog, k, x)) in lo for x in G.writes(prog, k)):
            s |= T
        for c in grp:
            if c <= k:
                continue
            for x, offs in G.reads(prog, c).items():
                v = G.version_read(prog, c, x)
                if v >= 1 and G.writer_of(prog, x, v) == k:
                    for p in pts[c]:
                        for d in offs:
                            s.add((p[0] + d[0], p[1] + d[1], p[2] + d[2]))
        pts[k] = s
    return {k: _bbox(pts[k]) for k in grp}, pts


def _bbox(s):
    if not s:
        return None
    lo = [-min(p[a] for p in s) for a in range(3)]
    hi = [max(p[a] for p in s) - (PT[a] - 1) for a in range(3)]
    return (tuple(lo), tuple(hi))


def load_boxes(prog: Program, grp: List[int], pts) -> Dict[Tuple[int, int], Optional[tuple]]:
    """Box read from HBM for each live-in version: U_{c reads it} E(c) (+) F_c(x)."""
    out = {}
    for (x, v) in live_in(prog, grp):
        s = set()
        for c in grp:
            offs = G.reads(prog, c).get(x)
            if offs is None or G.version_read(prog, c, x) != v:
                continue
            for p in pts[c]:
                for d in offs:
                    s.add((p[0] + d[0], p[1] + d[1], p[2] + d[2]))
        out[(x, v)] = _bbox(s)
    return out


def nonlocal_read(prog: Program, c: int, x: int, pts) -> bool:
    """Does kernel c read array x at any point outside the tile T (3D)?"""
    offs = G.reads(prog, c)[x]
    for p in pts[c]:
        for d in offs:
            q = (p[0] + d[0], p[1] + d[1], p[2] + d[2])
            if not all(0 <= q[a] < PT[a] for a in range(3)):
                return True
    return False


# ---------------------------------------------------------------- resource model (definition)
def rpn_depth(rpn) -> int:
    d = m = 0
    for ins in rpn:
        if ins.op in (OP_CONST, OP_PARAM, OP_LOAD):
            d += 1
        elif ins.op in (OP_NEG, OP_ABS, OP_SQRT):
            pass
        else:
            d -= 1
        m = max(m, d)
    return m


def _roundup(a, b):
    return (a + b - 1) // b * b


def schedule(prog: Program, grp: List[int], target: Target):
    """Streaming schedule of a group (lowering a3): per-kernel z delay D_k, SMEM-resident versions
    with their boxes, ring slots and bytes.  The definition the CUDA kernel must fit (R20)."""
    ext, pts = extended_regions(prog, grp)
    alive = [k for k in grp if ext[k] is not None]
    # delays: a consumer runs D_p + dz planes behind the producer of what it reads; with the delay
    # skew (R20c) a read at a nonzero xy offset runs U planes further behind
    D: Dict[int, int] = {}
    for k in alive:
        dk = 0
        for x, offs in G.reads(prog, k).items():
            v = G.version_read(prog, k, x)
            if v >= 1 and G.writer_of(prog, x, v) in alive:
                p = G.writer_of(prog, x, v)
                for d in offs:
                    lag = target.zunroll if (target.skew and (d[0] != 0 or d[1] != 0)) else 0
                    dk = max(dk, D[p] + d[2] + lag)
        D[k] = dk
    es = prog.es
    TX, TY = target.tile[0], target.tile[1]
    S = target.stages
    lin = live_in(prog, grp)
    lout = set(live_out(prog, grp))
    boxes = load_boxes(prog, grp, pts)
    res = []          # (kind, x, v, Wx, Hy, slots, bytes)
    for (x, v) in lin:
        rd = [(c, G.reads(prog, c)[x]) for c in alive if x in G.reads(prog, c) and G.version_read(prog, c, x) == v]
        if not rd:
            continue
        A = max(d[2] - D[c] for c, offs in rd for d in offs)
        B = min(d[2] - D[c] for c, offs in rd for d in offs)
        if not G.relaxed(prog, x):
            for b in alive:
                if x in G.writes(prog, b) and (x, G.version_written(prog, x=x, k=b)) in lout:
                    A = max(A, -D[b])
        span = A - B + 1
        slots = span + target.zunroll * S - 1      # U planes in use + U*(S-1) prefetched
        (lo, hi) = boxes[(x, v)]
        # the TMA box of a live-in starts on a 16-byte boundary in x (R20a): lower x extent rounded
        # up to a multiple of 16/es elements (toward +inf, also when negative)
        al = 16 // es
        lox = -((-lo[0]) // al) * al
        res.append(("in", x, v, TX + lox + hi[0], TY + lo[1] + hi[1], slots, A, B))
    for p in alive:
        for x in G.writes(prog, p):
            v = G.version_written(prog, p, x)
            rd = [(c, G.reads(prog, c)[x]) for c in alive if x in G.reads(prog, c)
                  and G.version_read(prog, c, x) == v]
            if not rd:
                continue
            span = max(D[c] - d[2] for c, offs in rd for d in offs) - D[p] + 1 + (target.zunroll - 1)
            (lo, hi) = ext[p]
            res.append(("mid", x, v, TX + lo[0] + hi[0], TY + lo[1] + hi[1], span, 0, 0))
    if target.ringunroll:   # ring depths rounded up to powers of two (stream loop unrolled, R20b)
        res = [r[:5] + (1 << (r[5] - 1).bit_length(),) + r[6:] for r in res]
    smem = 0
    for r in res:
        px = _roundup(r[3], 16 // es)
        plane = _roundup(px * r[4] * es, 128)
        smem += r[5] * plane
    smem += 8 * S + 128
    depth = max([rpn_depth(s.rpn) for k in grp for s in prog.kernels[k].stmts] + [1])
    # threads per CTA: one per register block (bx x by points) of the canvas when
    # the tile's blocks fit the target's thread count (<= 512); points per thread
    # P = pblock x zunroll x rounds (capped at 8)
    regions = [((TX + ext[k][0][0] + ext[k][1][0]), (TY + ext[k][0][1] + ext[k][1][1])) for k in alive]
    bx0, by0 = max(1, target.pblock[0]), max(1, target.pblock[1])
    # canvas = bounding box of all extended regions (per-axis max lo / max hi halo)
    cw = TX + max([ext[k][0][0] for k in alive] + [0]) + max([ext[k][1][0] for k in alive] + [0])
    ch = TY + max([ext[k][0][1] for k in alive] + [0]) + max([ext[k][1][1] for k in alive] + [0])
    maxb = (-(-cw // min(bx0, cw))) * (-(-ch // min(by0, ch))) if alive else 0
    nt = _roundup(maxb, 32)
    tb = (-(-TX // bx0)) * (-(-TY // by0))
    threads = nt if (tb <= target.threads and 32 <= nt <= 512) else target.threads
    rounds = 1
    for w, h in regions:
        bx, by = min(target.pblock[0], w), min(target.pblock[1], h)
        nb = (-(-w // bx)) * (-(-h // by))
        rounds = max(rounds, -(-nb // threads))
    P = min(8, target.pblock[0] * target.pblock[1] * target.zunroll * rounds)
    # register model (V8, R20 revised in round 2): the paper's Eq. 4/6,
    #   R_est = R_adr*U + RegFac*(es/4)*P*(ThrLD + depth)
    # R_adr = 32 per plane of a stream iteration, R_fetch = 0 (TMA), RegFac = 1 (no reuse, the upper
    # end of P:347's range), ThrLD = distinct (array, version, offset) loads a thread holds: the whole
    # group's on the canvas (one canvas point -- or one aligned pair -- per thread, rounds = 1), the
    # largest kernel's otherwise
    clo0 = max([ext[k][0][0] for k in alive] + [0])
    chi0 = max([ext[k][1][0] for k in alive] + [0])
    canvas = False
    if alive and tuple(target.pblock) == (1, 1):
        canvas = -(-(cw * ch) // threads) == 1
    if alive and tuple(target.pblock) == (2, 1) and target.zunroll == 1 and TX % 2 == 0 and prog.n[0] % 2 == 0:
        cwp = TX // 2 + (clo0 + 1) // 2 + (chi0 + 1) // 2
        canvas = -(-(cwp * ch) // threads) == 1
    loads = set()
    kmax = 0
    for k in alive:
        nk = 0
        for x, offs in G.reads(prog, k).items():
            v = G.version_read(prog, k, x)
            for d in offs:
                loads.add((x, v, tuple(d)))
                nk += 1
        kmax = max(kmax, nk)
    thrld = len(loads) if canvas else kmax
    regs = 32 * target.zunroll + (es // 4) * P * (thrld + depth)
    return dict(ext=ext, pts=pts, delay=D, res=res, smem=smem, regs=regs, alive=alive, threads=threads)


def regs_limit(threads: int) -> int:
    """Registers per thread an NT-thread CTA can have on B200 (Eq. 3 with one CTA per SM): the
    65536-register file is 4 sub-partitions of 16384, a CTA's warps spread over them, allocation in
    units of 8 registers per thread."""
    warps = -(-threads // 32)
    return min(255, 16384 // (-(-warps // 4) * 32) // 8 * 8)


# ---------------------------------------------------------------- validation
def quotient_order(prog: Program, plan: List[int]):
    """Kahn order of groups; ties -> smaller canonical label (smallest first kernel)."""
    gs = groups_of(plan)
    c = canonical(plan)
    m = len(gs)
    succ = [set() for _ in range(m)]
    indeg = [0] * m
    for (a, b, _, _) in G.edges(prog):
        if c[a] != c[b] and c[b] not in succ[c[a]]:
            succ[c[a]].add(c[b])
            indeg[c[b]] += 1
    order = []
    ready = sorted(g for g in range(m) if indeg[g] == 0)
    while ready:
        g = ready.pop(0)
        order.append(g)
        for h in sorted(succ[g]):
            indeg[h] -= 1
            if indeg[h] == 0:
                ready.append(h)
                ready.sort()
    return order if len(order) == m else None


def validate(prog: Program, plan: List[int], target: Target = Target()):
    """Returns (code, group, kernel_a, kernel_b, array) of the first violation, or (0,-1,-1,-1,-1)."""
    nk = len(prog.kernels)
    NONE = (V_OK, -1, -1, -1, -1)
    # V1
    if len(plan) != nk:
        return (V1_PARTITION, -1, -1, -1, -1)
    for k in range(nk):
        if plan[k] < 0:
            return (V1_PARTITION, -1, k, -1, -1)
    gs = groups_of(plan)
    c = canonical(plan)
    # V2
    if not (prog.flags & (1 << 2)):
        for g, grp in enumerate(gs):
            a = grp[0]
            for b in grp[1:]:
                if G.kinship(prog, a, b, grp) == 0:
                    return (V2_KINSHIP, g, a, b, -1)
    es_ = G.edges(prog)
    reach = G.closure(nk, es_)
    # V3
    for g, grp in enumerate(gs):
        for cc in range(nk):
            if c[cc] == g:
                continue
            src = [a for a in grp if reach[a][cc]]
            if src and any(reach[cc][b] for b in grp):
                return (V3_CONVEX, g, min(src), cc, -1)
    # V4
    m = len(gs)
    q = [(c[a], c[b]) for (a, b, _, _) in es_ if c[a] != c[b]]
    qr = G.closure(m, q)
    for g in range(m):
        if qr[g][g]:
            return (V4_CYCLE, g, -1, -1, -1)
    scheds = [schedule(prog, grp, target) for grp in gs]
    # V5
    for g, grp in enumerate(gs):
        pts = scheds[g]["pts"]
        lin = set(live_in(prog, grp))
        lout = set(live_out(prog, grp))
        for b in grp:
            for x in sorted(G.writes(prog, b)):
                if G.relaxed(prog, x) or (x, G.version_written(prog, b, x)) not in lout:
                    continue
                for a in grp:
                    if x not in G.reads(prog, a):
                        continue
                    if (x, G.version_read(prog, a, x)) not in lin:
                        continue
                    if nonlocal_read(prog, a, x, pts):
                        return (V5_HAZARD, g, a, b, x)
    # V6
    for g, grp in enumerate(gs):
        ext, pts = scheds[g]["ext"], scheds[g]["pts"]
        boxes = load_boxes(prog, grp, pts)
        for (x, v) in sorted(boxes):
            bb = boxes[(x, v)]
            if bb is None:
                continue
            lo, hi = bb
            for a in range(3):
                wrap = prog.bc[a] == BC_PERIODIC or (target.internal_axes >> a) & 1
                if wrap and max(lo[a], hi[a]) > prog.ghost[a]:
                    return (V6_HALO, g, -1, -1, x)
                if a < 2 and max(lo[a], hi[a]) > target.max_halo:
                    return (V6_HALO, g, -1, -1, x)
        for k in grp:
            if ext[k] is None:
                continue
            lo, hi = ext[k]
            if max(lo[0], hi[0], lo[1], hi[1]) > target.max_halo:
                return (V6_HALO, g, k, -1, -1)
    # V7, V8
    for g in range(m):
        if scheds[g]["smem"] > target.smem_per_block:
            return (V7_SMEM, g, -1, -1, -1)
    for g in range(m):   # Eq. 2 (R_T <= R_Max) and Eq. 3 with one CTA per SM (per register-file quadrant)
        if scheds[g]["regs"] > min(target.regs_per_thread_max, regs_limit(scheds[g]["threads"])):
            return (V8_REGS, g, -1, -1, -1)
    return NONE


# ---------------------------------------------------------------- bytes (O-6) and projection (O-9)
def bytes_by_counting(prog: Program, plan: List[int]):
    """Replay the plan group by group on the interior with per-(version, point) flags:
    a read is counted the first time the group touches a version it does not produce, a write
    when the group's version is live-out.  Eq. 11's LD/ST counts, in bytes."""
    import numpy as np
    gs = groups_of(plan)
    nx, ny, nz = prog.n
    out = []
    for grp in gs:
        read_flags: Dict[Tuple[int, int], np.ndarray] = {}
        rb = 0
        for k in grp:
            for x in G.reads(prog, k):
                v = G.version_read(prog, k, x)
                if v >= 1 and G.writer_of(prog, x, v) in grp:
                    continue
                f = read_flags.setdefault((x, v), np.zeros((nz, ny, nx), dtype=bool))
                rb += int((~f).sum())
                f[:] = True
        wb = 0
        for (x, v) in live_out(prog, grp):
            wb += nx * ny * nz
        out.append((rb * prog.es, wb * prog.es))
    return out


def project(prog: Program, plan: List[int], target: Target = Target()):
    """Codeless upper bound (Eq. 11): t(G) = compulsory bytes / peak bandwidth,
    total = left fold in canonical group order."""
    per = bytes_by_counting(prog, plan)
    tot_b = 0
    tot_t = 0.0
    res = []
    for (r, w) in per:
        t = float(r + w) / target.hbm_bytes_per_s
        res.append((r, w, t))
        tot_b += r + w
        tot_t += t
    return res, tot_b, tot_t


def unfused_bytes(prog: Program) -> int:
    return project(prog, list(range(len(prog.kernels))))[1]
