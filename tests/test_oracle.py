"""Pins of the oracle against what the paper and mathematics fix (no GPU).

Each test names the pin: closed forms, invariants, brute force on tiny inputs,
paper worked examples (tests/golden), counting identities.
"Oracle pins".
"""
import itertools
import json
import os

import numpy as np
import pytest

from oracle import enum as En
from oracle import graph as G
from oracle import interp
from oracle import legality as L
from oracle import tilesim as TS
from workloads import data as D
from workloads import programs as P
from workloads.program import (ARRAY_OUTPUT, BC_FROZEN, BC_PERIODIC, DT_F32, DT_F64, Builder,
                               PROG_RELAX_ALL, PROG_RELAX_EXPANDABLE, emin, emax, eabs, esqrt)

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def bits(a):
    return a.view(np.uint32 if a.dtype == np.float32 else np.uint64)


def interior(prog, a, shrink=0):
    g = prog.ghost
    s = shrink
    return a[g[2] + s:a.shape[0] - g[2] - s, g[1] + s:a.shape[1] - g[1] - s, g[0] + s:a.shape[2] - g[0] - s]


# ------------------------------------------------------------------ O-1 closed forms
def test_L7_of_quadratic_is_12_and_chain_closed_form():
    """App. B: 7-pt Laplacian of i^2+2j^2+3k^2 is 2+4+6 = 12; L7 of a constant is 0;
    K3 halves u so step 2 gives 6 away from the frozen boundary."""
    prog = P.tiny()
    inp = D.quadratic(prog)
    r1 = interp.run(prog, inp, 1)
    assert np.all(interior(prog, r1["v"]) == 12.0)
    assert np.all(interior(prog, r1["w"], 1) == 0.0)
    r2 = interp.run(prog, inp, 2)
    assert np.all(interior(prog, r2["v"], 1) == 6.0)
    assert np.all(interior(prog, r2["w"], 2) == 0.0)


def _single(prog_builder_fn, n=(12, 10, 9), ghost=4, dtype=DT_F64):
    b = Builder("cf", dtype, n, (ghost,) * 3, (BC_FROZEN,) * 3)
    u = b.array("u")
    o = b.array("o")
    b.kernel("k", (o, prog_builder_fn(u)))
    return b.build()


def test_13pt_27pt_25pt_closed_forms():
    """App. B: x12 13-pt of i^2 = 24; x30 27-pt isotropic of x^2+2y^2+3z^2 = 360;
    x5040 25-pt radius-4 of i^2 = 10080 per axis; all stencils annihilate linear fields."""
    def w13(u):
        t = []
        for a in range(3):
            for off, w in zip((-2, -1, 0, 1, 2), (-1.0, 16.0, -30.0, 16.0, -1.0)):
                d = [0, 0, 0]; d[a] = off
                t.append(w * u[tuple(d)])
        acc = t[0]
        for x in t[1:]:
            acc = acc + x
        return acc

    def w27(u):
        terms = []
        for dz in (-1, 0, 1):
            for dy in (-1, 0, 1):
                for dx in (-1, 0, 1):
                    nz = (dx != 0) + (dy != 0) + (dz != 0)
                    w = {0: -128.0, 1: 14.0, 2: 3.0, 3: 1.0}[nz]
                    terms.append(w * u[dx, dy, dz])
        acc = terms[0]
        for x in terms[1:]:
            acc = acc + x
        return acc

    cases = [(w13, lambda i, j, k: i * i, 24.0 * 1), (w13, lambda i, j, k: i * i + 2 * j * j + 3 * k * k, 24.0 * 6),
             (w27, lambda i, j, k: i * i + 2 * j * j + 3 * k * k, 360.0),
             (lambda u: P.L25(u, 1.0), lambda i, j, k: i * i, 10080.0),
             (lambda u: P.L25(u, 1.0), lambda i, j, k: i * i + 2 * j * j + 3 * k * k, 60480.0)]
    for st, field, expect in cases:
        prog = _single(st)
        i, j, k = D.coords(prog)
        inp = {"u": field(i, j, k).astype(np.float64), "o": np.zeros(prog.padded_shape())}
        out = interp.run(prog, inp, 1)
        assert np.all(interior(prog, out["o"]) == expect), (st, expect)
        lin = {"u": (3 * i - 5 * j + 7 * k + 11).astype(np.float64), "o": inp["o"]}
        assert np.all(interior(prog, interp.run(prog, lin, 1)["o"]) == 0.0)


def test_linear_field_preserved_bit_exactly():
    """u <- u + nu*L7(u) leaves a linear field unchanged (L7 of linear = 0, exact in fp64)."""
    b = Builder("lin", DT_F64, (10, 9, 8), (1, 1, 1), (BC_FROZEN,) * 3)
    u = b.array("u")
    t = b.array("t")
    nu = b.param(0.1)
    b.kernel("lap", (t, P.L7(u)))
    b.kernel("upd", (u, u.c + nu * t.c))
    prog = b.build()
    i, j, k = D.coords(prog)
    u0 = (2.0 * i + 3.0 * j - k + 0.5).astype(np.float64)
    out = interp.run(prog, {"u": u0, "t": np.zeros_like(u0)}, 5)
    assert np.array_equal(bits(out["u"]), bits(u0))


def test_periodic_flux_form_conserves_exactly():
    """Invariant: periodic flux-form update phi -= (F - F[-1]) with integer data and weights
    conserves sum(phi) exactly (telescoping sum; all values are integers < 2^53)."""
    b = Builder("cons", DT_F64, (8, 6, 5), (2, 2, 2), (BC_PERIODIC,) * 3)
    phi = b.array("phi")
    F = b.array("F")
    b.kernel("flux", (F, 3.0 * phi.c - phi[1, 0, 0] + 2.0 * phi[0, -1, 0]))
    b.kernel("upd", (phi, phi.c - (F.c - F[-1, 0, 0])))
    prog = b.build()
    rng = np.random.default_rng(7)
    p0 = rng.integers(-50, 50, size=prog.padded_shape()).astype(np.float64)
    out = interp.run(prog, {"phi": p0, "F": np.zeros_like(p0)}, 3)
    assert interior(prog, out["phi"]).sum() == interior(prog, p0).sum()


def test_periodic_shift_identity_after_n_steps():
    """A periodic shift by one cell along x returns the identity after nx steps."""
    b = Builder("shift", DT_F32, (7, 5, 4), (1, 1, 1), (BC_PERIODIC,) * 3)
    a = b.array("a")
    t = b.array("t")
    b.kernel("s", (t, a[-1, 0, 0]))
    b.kernel("c", (a, t.c))
    prog = b.build()
    a0 = D.uniform(prog, 3)["a"]
    out = interp.run(prog, {"a": a0, "t": np.zeros_like(a0)}, 7)
    assert np.array_equal(bits(interior(prog, out["a"])), bits(interior(prog, a0)))


def test_jacobi_sweep_equals_textbook_slicing():
    """Special case: one 7-pt Jacobi sweep equals the textbook numpy slicing expression."""
    b = Builder("jac", DT_F64, (9, 8, 7), (1, 1, 1), (BC_FROZEN,) * 3)
    u = b.array("u")
    o = b.array("o")
    b.kernel("j", (o, (u[-1, 0, 0] + u[1, 0, 0] + u[0, -1, 0] + u[0, 1, 0] + u[0, 0, -1] + u[0, 0, 1]) * (1.0 / 6.0)))
    prog = b.build()
    inp = D.uniform(prog, 4)
    out = interp.run(prog, inp, 1)
    U = inp["u"]
    ref = (U[1:-1, 1:-1, :-2] + U[1:-1, 1:-1, 2:] + U[1:-1, :-2, 1:-1] + U[1:-1, 2:, 1:-1]
           + U[:-2, 1:-1, 1:-1] + U[2:, 1:-1, 1:-1]) * (1.0 / 6.0)
    assert np.array_equal(bits(interior(prog, out["o"])), bits(ref))


def test_brute_force_scalar_evaluation_fp32():
    """Brute force on tiny inputs: the vectorised interpreter equals a point-by-point loop
    with numpy float32 scalars (checks indexing, boundary rules and op order)."""
    prog = P.random_program(11, nk=4, na=4, n=(4, 3, 3), dtype=DT_F32,
                            bc=(BC_PERIODIC, BC_FROZEN, BC_PERIODIC))
    inp = D.uniform(prog, 5)
    out = interp.run(prog, inp, 1)
    arrs = [inp[nm].copy() for nm, _ in prog.arrays]
    g = prog.ghost
    n = prog.n

    def idx(a, q):
        if prog.bc[a] == BC_PERIODIC:
            q = q % n[a]
        return q + g[a]

    with np.errstate(all="ignore"):
        for kern in prog.kernels:
            new = []
            for s in kern.stmts:
                res = np.zeros((n[2], n[1], n[0]), dtype=np.float32)
                for z, y, x in itertools.product(range(n[2]), range(n[1]), range(n[0])):
                    st = []
                    for ins in s.rpn:
                        if ins.op == 0:
                            st.append(np.float32(ins.imm))
                        elif ins.op == 1:
                            st.append(np.float32(prog.params[ins.arg]))
                        elif ins.op == 2:
                            st.append(arrs[ins.arg][idx(2, z + ins.d[2]), idx(1, y + ins.d[1]), idx(0, x + ins.d[0])])
                        elif ins.op in (9, 10, 11):
                            a = st.pop()
                            st.append({9: lambda: -a, 10: lambda: abs(a), 11: lambda: np.sqrt(a)}[ins.op]())
                        else:
                            bb, aa = st.pop(), st.pop()
                            st.append({3: lambda: aa + bb, 4: lambda: aa - bb, 5: lambda: aa * bb,
                                       6: lambda: aa / bb, 7: lambda: bb if bb < aa else aa,
                                       8: lambda: bb if aa < bb else aa}[ins.op]())
                    res[z, y, x] = st[0]
                new.append((s.out, res))
            for o, r in new:
                arrs[o][g[2]:g[2] + n[2], g[1]:g[1] + n[1], g[0]:g[0] + n[0]] = r
    for i, (nm, _) in enumerate(prog.arrays):
        assert np.array_equal(bits(out[nm]), bits(arrs[i])), nm


def test_min_max_select_semantics_special_values():
    """R16: MIN(a,b) := (b<a)?b:a and MAX(a,b) := (a<b)?b:a, including NaN and signed zeros."""
    b = Builder("mm", DT_F64, (4, 1, 1), (0, 0, 0), (BC_FROZEN,) * 3)
    A, B_, o1, o2 = b.array("a"), b.array("b"), b.array("mn"), b.array("mx")
    b.kernel("k", (o1, emin(A.c, B_.c)), (o2, emax(A.c, B_.c)))
    prog = b.build()
    a = np.array([np.nan, 0.0, -0.0, 1.0]).reshape(1, 1, 4)
    bb = np.array([1.0, -0.0, 0.0, np.nan]).reshape(1, 1, 4)
    out = interp.run(prog, {"a": a, "b": bb, "mn": np.zeros_like(a), "mx": np.zeros_like(a)}, 1)
    exp_mn = [y if y < x else x for x, y in zip(a.ravel(), bb.ravel())]
    exp_mx = [y if x < y else x for x, y in zip(a.ravel(), bb.ravel())]
    assert np.array_equal(bits(out["mn"].ravel()), bits(np.array(exp_mn)))
    assert np.array_equal(bits(out["mx"].ravel()), bits(np.array(exp_mx)))


def test_constants_rounded_to_fp32():
    """CONST is rounded to the program dtype before use: 0.1f*3 != 0.1*3 in fp64."""
    b = Builder("c", DT_F32, (2, 1, 1), (0, 0, 0), (BC_FROZEN,) * 3)
    a, o = b.array("a"), b.array("o")
    b.kernel("k", (o, a.c * 0.1))
    prog = b.build()
    x = np.full((1, 1, 2), 3.0, dtype=np.float32)
    out = interp.run(prog, {"a": x, "o": np.zeros_like(x)}, 1)
    assert out["o"].dtype == np.float32
    assert out["o"][0, 0, 0] == np.float32(3.0) * np.float32(0.1)


# ------------------------------------------------------------------ O-2/3/4 graphs
def test_tiny_edges_classes_liveness():
    prog = P.tiny()
    assert G.edges(prog) == [(0, 1, G.RAW, 1), (0, 2, G.WAR, 0)]
    assert [G.array_class(prog, x) for x in range(3)] == [G.CLS_RW, G.CLS_RW, G.CLS_WO]
    assert [G.step_live(prog, x) for x in range(3)] == [True, False, True]


def test_fig3_table2_golden():
    gold = json.load(open(os.path.join(GOLD, "table2_fig3.json")))
    prog = P.fig3()
    kn = [k.name for k in prog.kernels]
    an = [a for a, _ in prog.arrays]
    K = lambda s: kn.index(s)
    A = lambda s: an.index(s)
    for arr, ks in gold["sharing_set"].items():
        assert sorted(kn[k] for k in G.sharing_set(prog, A(arr))) == sorted(ks)
    for name, pv in gold["pivot"].items():
        grp = [K(s) for s in pv["group"]]
        assert sorted(an[x] for x in G.pivot(prog, grp)) == sorted(pv["arrays"])
    for kk in gold["kinship"]:
        assert G.kinship(prog, K(kk["a"]), K(kk["b"]), [K(s) for s in kk["group"]]) == kk["degree"]
    for tl in gold["thread_load"]:
        assert len(prog.kernels[K(tl["kernel"])].reads()[A(tl["array"])]) == tl["value"]
    exp = sorted((K(a), K(b), G.RAW, A(x)) for a, b, x in gold["precedence_edges_RAW"])
    assert G.edges(prog) == exp
    plan = [0] * len(kn)
    for gi, (_, ks) in enumerate(sorted(gold["fused_plans_of_figure"].items())):
        for s in ks:
            plan[K(s)] = gi
    assert L.validate(prog, plan)[0] == L.V_OK   # the paper's own fusion is legal


def test_weather_classes_and_expandable_flux():
    """QFLX_* are written by 5 kernels each -> expandable (like QFLX in P:53)."""
    prog = P.weather(n=(8, 8, 8))
    an = [a for a, _ in prog.arrays]
    for s in ("QFLX_X", "QFLX_Y", "QFLX_Z", "DMOMX"):
        assert G.array_class(prog, an.index(s)) == G.CLS_EXPANDABLE
    for s in ("DENS0", "CORI"):
        assert G.array_class(prog, an.index(s)) == G.CLS_RO
    assert len(prog.kernels) == 44 and len(prog.arrays) == 31


@pytest.mark.parametrize("seed", range(12))
def test_canonical_edges_preserve_closure(seed):
    """Nearest-access canonical edges have the same transitive closure as all pairwise hazards."""
    for flags in (0, PROG_RELAX_EXPANDABLE, PROG_RELAX_ALL):
        prog = P.random_program(seed, nk=7, na=4, flags=flags)
        nk = len(prog.kernels)
        c1 = G.closure(nk, G.edges(prog))
        c2 = G.closure(nk, list(G.all_pairs_hazards(prog)))
        assert c1 == c2


# ------------------------------------------------------------------ O-5/O-8 legality
@pytest.mark.parametrize("nk", [3, 4, 5, 6])
def test_brute_force_counts(nk):
    """pointwise chain: 2^(n-1) (contiguous segments); shared RO array: Bell(n); disjoint: 1."""
    assert len(En.legal_plans(P.pointwise_chain(nk))) == 2 ** (nk - 1)
    assert len(En.legal_plans(P.shared_readonly(nk))) == En.bell(nk)
    assert len(En.legal_plans(P.disjoint(nk))) == 1
    assert sum(1 for _ in En.restricted_growth(nk)) == En.bell(nk)


def test_tiny_legality_table():
    prog = P.tiny()
    got = {tuple(p): L.validate(prog, p) for p in En.restricted_growth(3)}
    assert got[(0, 1, 2)][0] == L.V_OK
    assert got[(0, 0, 1)][0] == L.V_OK
    assert got[(0, 0, 0)] == (L.V5_HAZARD, 0, 0, 2, 0)     # K1 reads u at offsets, K3 overwrites u
    assert got[(0, 1, 0)] == (L.V5_HAZARD, 0, 0, 2, 0)
    assert got[(0, 1, 1)][0] == L.V2_KINSHIP                # K2, K3 share no array
    relaxed = P.tiny(flags=PROG_RELAX_ALL)
    assert len(En.legal_plans(relaxed)) == 4
    assert len(En.legal_plans(P.tiny(flags=PROG_RELAX_EXPANDABLE))) == 2


def test_cycle_and_convexity():
    """R4: convex groups can still deadlock: A->B, C->D with {A,D}, {B,C}."""
    b = Builder("cyc", DT_F64, (4, 4, 4), (1, 1, 1), (BC_FROZEN,) * 3)
    s = b.array("s")
    x = b.array("x")
    y = b.array("y")
    t = b.array("t")
    b.kernel("A", (x, s.c + 1.0))
    b.kernel("B", (y, x.c * s.c))
    b.kernel("C", (t, s.c - 1.0))
    b.kernel("D", (s, t.c * 2.0 + s.c))
    prog = b.build()
    # edges: A->B (RAW x), C->D (RAW t), and WAR s from A,B,C to D
    v = L.validate(prog, [0, 1, 1, 0])
    assert v[0] in (L.V3_CONVEX, L.V4_CYCLE)
    b2 = Builder("cyc2", DT_F64, (4, 4, 4), (1, 1, 1), (BC_FROZEN,) * 3)
    p, q, r1, r2, sh = b2.array("p"), b2.array("q"), b2.array("r1"), b2.array("r2"), b2.array("sh", 2)
    b2.kernel("A", (p, sh.c + 1.0))
    b2.kernel("B", (q, p.c + sh.c))
    b2.kernel("C", (r1, sh.c * 3.0))
    b2.kernel("D", (r2, r1.c + sh.c))
    prog2 = b2.build()
    assert L.validate(prog2, [0, 1, 1, 0])[0] == L.V4_CYCLE
    assert L.validate(prog2, [0, 0, 1, 1])[0] == L.V_OK


@pytest.mark.parametrize("seed", range(16))
def test_tile_simulator_pins_V5(seed):
    """Semantic pin (O-7): for plans passing V1-V4, V5 says legal  <=>  every tile order of the
    fused execution reproduces the unfused interpreter bit for bit."""
    rng = np.random.default_rng(100 + seed)
    bc = tuple(int(x) for x in rng.integers(0, 2, size=3))
    flags = [0, PROG_RELAX_EXPANDABLE, PROG_RELAX_ALL][seed % 3]
    prog = P.random_program(seed, nk=4, na=4, n=(6, 4, 4), bc=bc, flags=flags)
    inp = D.uniform(prog, seed)
    ref = interp.run(prog, inp, 2)
    tile = (3, 2, 2)
    nt = TS.n_tiles(prog, tile)
    orders = [list(range(nt)), list(reversed(range(nt)))] + [list(rng.permutation(nt)) for _ in range(3)]
    live = [nm for x, (nm, _) in enumerate(prog.arrays) if G.step_live(prog, x) or not G.writers(prog, x)]
    checked = 0
    for plan in En.restricted_growth(len(prog.kernels)):
        v = L.validate(prog, plan)
        if v[0] in (L.V1_PARTITION, L.V2_KINSHIP, L.V3_CONVEX, L.V4_CYCLE):
            continue
        ok_all = True
        for order in orders:
            out = TS.run_fused(prog, plan, inp, 2, tile, order)
            if not all(np.array_equal(bits(out[nm]), bits(ref[nm])) for nm in live):
                ok_all = False
                break
        if v[0] == L.V5_HAZARD:
            assert not ok_all, (plan, v)
        else:
            assert ok_all, (plan, v)
        checked += 1
    assert checked >= 1


def test_tile_simulator_pins_V6_ghost_rule():
    """Semantic pin of V6 (O-7, ghost-limited mode): periodic neighbours are read only through the
    stored ghost layer (width `ghost`, refreshed before every group as the device does).  For plans
    passing V1-V5: V6 legal  <=>  the fused execution reproduces the unfused interpreter bit for
    bit; a plan whose accumulated input halo exceeds the ghost width reads past the ghost layer."""
    n_v6 = n_ok = 0
    for seed in range(12):
        rng = np.random.default_rng(500 + seed)
        bc = (1, 1, int(rng.integers(0, 2)))
        flags = [0, PROG_RELAX_EXPANDABLE, PROG_RELAX_ALL][seed % 3]
        prog = P.random_program(900 + seed, nk=4, na=4, n=(6, 5, 4), bc=bc, flags=flags, max_r=1)
        inp = D.uniform(prog, seed)
        ref = interp.run(prog, inp, 2)
        live = [nm for x, (nm, _) in enumerate(prog.arrays) if G.step_live(prog, x) or not G.writers(prog, x)]
        for plan in En.restricted_growth(len(prog.kernels)):
            v = L.validate(prog, plan)
            if v[0] not in (L.V_OK, L.V6_HALO):
                continue
            out = TS.run_fused(prog, plan, inp, 2, (3, 2, 2), "snapshot", ghost_limited=True)
            # periodic ghost layers hold refreshed wraps here (the device's too, R9): compare the
            # interior and the frozen ghosts
            m = np.ones(prog.padded_shape(), bool)
            for a in range(3):
                if prog.bc[a] == 1:
                    sl = [slice(None)] * 3
                    sl[2 - a] = np.r_[0:prog.ghost[a], prog.n[a] + prog.ghost[a]:prog.n[a] + 2 * prog.ghost[a]]
                    m[tuple(sl)] = False
            exact = all(np.array_equal(bits(out[nm][m]), bits(ref[nm][m])) for nm in live)
            assert exact == (v[0] == L.V_OK), (seed, plan, v)
            n_v6 += v[0] == L.V6_HALO
            n_ok += v[0] == L.V_OK
    assert n_v6 >= 5 and n_ok >= 20, (n_v6, n_ok)


def test_tile_simulator_fig3_and_tiny():
    for prog, plan, nsteps in ((P.fig3(n=(8, 6, 4)), P.FIG3_PLAN_XY, 1), (P.tiny(n=(8, 8, 8)), [0, 0, 1], 3)):
        inp = D.inputs_for(prog, 3)
        ref = interp.run(prog, inp, nsteps)
        for order in ("snapshot", list(range(TS.n_tiles(prog, (4, 3, 2))))):
            out = TS.run_fused(prog, plan, inp, nsteps, (4, 3, 2), order)
            for x, (nm, _) in enumerate(prog.arrays):
                if G.step_live(prog, x) or not G.writers(prog, x):
                    assert np.array_equal(bits(out[nm]), bits(ref[nm])), nm


def test_weather_greedy_plan_shape_legal():
    """A hand plan of App. A.4 (diag, 5x{flux3+div}, PG+Coriolis, LAP chains, RK singles)."""
    prog = P.weather(n=(8, 8, 8))
    plan = weather_hand_plan(prog)
    assert L.validate(prog, plan)[0] == L.V_OK
    fused = L.project(prog, plan)[1] // (prog.es * prog.npts)
    assert fused < 142


from workloads.programs import weather_hand_plan  # noqa: E402


# ------------------------------------------------------------------ O-6 bytes / O-9 projection
def test_bytes_hand_counts():
    t = P.tiny()
    N = t.npts * 4
    assert L.project(t, [0, 1, 2])[1] == 6 * N == 786432
    assert L.project(t, [0, 0, 1])[1] == 4 * N == 524288
    f = P.fig3()
    assert L.unfused_bytes(f) == 18 * f.npts * 8
    assert L.project(f, P.FIG3_PLAN_XY)[1] == 13 * f.npts * 8
    w = P.weather(n=(8, 8, 8))
    assert L.unfused_bytes(w) == 142 * w.npts * 8       # counted by hand from App. A.4


@pytest.mark.parametrize("seed", range(10))
def test_bytes_closed_form_and_monotone(seed):
    """counting == es*N*(|LiveIn|+|LiveOut|) per group; unfused == sum_k(|R_k|+|W_k|) when every
    write is read or final; coarsening a partition never increases bytes; t == bytes/BW."""
    prog = P.random_program(seed, nk=5, na=4)
    tgt = L.Target()
    for plan in En.restricted_growth(5):
        per = L.bytes_by_counting(prog, plan)
        for grp, (r, w) in zip(L.groups_of(plan), per):
            assert r == prog.es * prog.npts * len(L.live_in(prog, grp))
            assert w == prog.es * prog.npts * len(L.live_out(prog, grp))
        res, tb, tt = L.project(prog, plan, tgt)
        acc = 0.0
        for (r, w, t) in res:
            assert t == float(r + w) / tgt.hbm_bytes_per_s
            acc += t
        assert tt == acc
    singles = L.project(prog, list(range(5)))[1]
    for plan in En.restricted_growth(5):
        assert L.project(prog, plan)[1] <= singles
    dead = any(not G.readers_of_version(prog, x, G.version_written(prog, k, x))
               and G.version_written(prog, k, x) != len(G.writers(prog, x))
               for k in range(5) for x in G.writes(prog, k))
    if not dead:
        naive = sum(len(G.reads(prog, k)) + len(G.writes(prog, k)) for k in range(5)) * prog.npts * prog.es
        assert singles == naive


def test_resource_model_worked_example():
    """V7 model (R20), hand-worked for tiny {K1,K2}, fp32, tile 32x16, S=2 stages, U=2 planes/iteration:
    delays D(K1)=0, D(K2)=1 (K2 reads v at dz=+1).
    u (live-in): box x extent below T 2 -> 4 (16-byte TMA start, R20a), width 32+4+2=38 -> row 40,
      height 20, A=1-0=1, B=-1-0=-1 -> span 3, slots 3+U*S-1=6, plane roundup(40*20*4,128)=3200
    v (in-group): box 34x18 -> row 36, span (1-(-1))-0+1 = 3, slots 3+(U-1)=4,
      plane roundup(36*18*4,128)=2688
    total = 6*3200 + 4*2688 + 8*2 + 128 = 30096;  with U=1: 4*3200 + 3*2688 + 144 = 21008."""
    s = L.schedule(P.tiny(), [0, 1], L.Target(tile=(32, 16, 0), zunroll=2))
    assert s["delay"] == {0: 0, 1: 1}
    assert s["smem"] == 6 * 3200 + 4 * 2688 + 16 + 128 == 30096
    assert L.schedule(P.tiny(), [0, 1], L.Target(tile=(32, 16, 0), zunroll=1))["smem"] == 21008


def test_L25_radius4_stencil_closed_form_through_stress_program():
    """Config 5 kernels: L25 (x5040 weights / 5040) of i^2+2j^2+3k^2 is 2+4+6 = 12 exactly in fp64
    (power-of-two-free but exact: integer weights, products < 2^53), so t1 = 12 and t2 = 0 inside."""
    prog = P.stress(m=1, n=(20, 20, 20))
    i, j, k = D.coords(prog)
    f = (i * i + 2 * j * j + 3 * k * k).astype(np.float64)
    inp = {"f0": f, "t1_0": np.zeros_like(f), "t2_0": np.zeros_like(f)}
    out = interp.run(prog, inp, 1)
    t1 = interior(prog, out["t1_0"])[:, 4:-4, 4:-4]        # away from the periodic xy wrap
    assert np.allclose(t1, 12.0, rtol=0, atol=1e-9)
    t2 = interior(prog, out["t2_0"])[4:-4, 8:-8, 8:-8]      # L25 of a constant is 0 (frozen z ghosts differ)
    assert np.allclose(t2, 0.0, rtol=0, atol=1e-9)


def test_paper_eq8_worked_example_golden():
    """NEXT-2 pin: the paper's worked example: B_Sh = 688 exactly, and the printed
    formula 688*14*202/(8*128*64) = 29.688 GFLOPS (75.37 % of 39.39; the paper prints 75.8 %)."""
    from oracle import paper_model
    gold = json.load(open(os.path.join(GOLD, "eq8_worked_example.json")))
    r = paper_model.project(**gold["inputs"])
    assert r["h_th"] == 1
    assert r["b_sh"] == gold["printed"]["b_sh"]
    assert r["p_membound_gflops"] == 688 * 14 * 202 / (8 * 128 * 64) == gold["derived_from_printed_formula"]["p_membound_gflops"]
    assert round(100 * r["p_membound_gflops"] / gold["printed"]["roofline_gflops"], 2) == gold["derived_from_printed_formula"]["percent"]


def test_paper_eq10_hand_calculation_golden():
    """NEXT-2 pin of T_pro (Eq. 10) under reading R12, against the hand calculation in
    tests/golden/eq10_hand_calc.json (exact rational arithmetic written out step by step)."""
    from oracle import paper_model
    gold = json.load(open(os.path.join(GOLD, "eq10_hand_calc.json")))
    i = gold["inputs"]
    r = paper_model.project(**{k: i[k] for k in ("t_b", "blocks_smx", "thr", "blocks", "hal", "halo", "shared_arrays",
                                                 "smx", "gmem_bw_gbs", "elem_bytes", "fl_unfused_sum", "flop_halo_sum")})
    e = gold["expected"]
    assert r["h_th"] == e["h_th"] and r["b_sh"] == e["b_sh"] and r["b_eff"] == e["b_eff"]
    assert r["p_membound_gflops"] == e["p_membound_gflops"]
    assert r["t_pro_s"] == pytest.approx(e["t_pro_s"], rel=1e-15, abs=0)
    # no halo layer (c = 0): T_pro is the unfused FLOPs over P_MemBound with B_Sh = T_B*Blocks/|ShrLst|
    r0 = paper_model.project(**dict({k: i[k] for k in ("t_b", "blocks_smx", "thr", "blocks", "hal", "shared_arrays",
                                                       "smx", "gmem_bw_gbs", "elem_bytes", "fl_unfused_sum",
                                                       "flop_halo_sum")}, halo=0))
    assert r0["b_sh"] == 86 * 32 / 2 and r0["t_pro_s"] < r["t_pro_s"]


def test_suite_generator_thread_load_and_sharing_sets():
    """NEXT-3 generator: the average thread load (distinct offsets per kernel-array read, R10) follows
    Table V's parameter and every sharing set stays within 2..8 kernels."""
    from oracle import graph as Gr
    for nk, load in ((30, 4), (60, 8), (100, 12)):
        d = P.gen_suite(n_kernels=nk, n_arrays=2 * nk, seed=1, n=(8, 8, 4), load=load, max_tries=2000)
        loads = [len(offs) for k in range(nk) for offs in Gr.reads(d, k).values()]
        assert abs(sum(loads) / len(loads) - load) < 1.0, (nk, load, sum(loads) / len(loads))
        users = {}
        for k in range(nk):
            for x in set(Gr.reads(d, k)) | set(Gr.writes(d, k)):
                users.setdefault(x, set()).add(k)
        assert all(len(u) <= 8 for u in users.values())
