"""GPU parity of the round-2 features and edge cases, through the C ABI, against the oracle.

* every opcode (MIN/MAX/ABS/SQRT/DIV/NEG included) on NaN, +-0, +-inf, x/0 and sqrt(<0) inputs,
  every legal plan: IEEE results equal the oracle's bit for bit where not NaN, NaN exactly where
  the oracle has NaN (reading R16b: NaN payloads are not specified by IEEE 754 for arithmetic);
* periodic ghost copies written by the producing groups (ghostwrite) in the pair canvas: no
  ghost-fill launches, same results;
* the one-call interface kf_run (per-plan executor cache) and kf_scratch_bytes;
* kf_exec_invalidate after changing FROZEN ghost values under the same pointers;
* domain decomposition with a periodic z axis and the exchange/compute overlap on,
  and the dist CUDA graph vs eager replay."""
import numpy as np
import pytest

from oracle import enum as En
from oracle import interp
from workloads import data as D
from workloads import programs as P
from workloads.program import (BC_FROZEN, BC_PERIODIC, DT_F32, DT_F64, PROG_RELAX_ALL, Builder, eabs, emax, emin,
                               esqrt)

from .gpu_util import bits, defined_cells, kept_arrays, run_kf

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a GPU", allow_module_level=True)

import paper_conf_sc_wahibm14_b200 as kf  # noqa: E402


def compare_nan(desc, got, ref):
    """Bitwise on non-NaN cells, NaN exactly where the oracle has NaN (R16b)."""
    bad = []
    mask = defined_cells(desc)
    for nm in kept_arrays(desc):
        g, o = got[nm][mask], ref[nm][mask]
        gn, on = np.isnan(g), np.isnan(o)
        if not np.array_equal(gn, on):
            bad.append((nm, "nan-mask", int(np.sum(gn != on))))
            continue
        if not np.array_equal(bits(g[~gn]), bits(o[~on])):
            bad.append((nm, "bits", int(np.sum(bits(g[~gn]) != bits(o[~on])))))
    return bad


def special_program(dtype, bc=(BC_PERIODIC, BC_FROZEN, BC_FROZEN)):
    b = Builder("ops", dtype, (40, 12, 6), (1, 1, 1), bc)
    a, bb, c, d, e = (b.array(n) for n in ("a", "b", "c", "d", "e"))
    b.kernel("K1", (c, emin(a.c, bb[1, 0, 0]) + emax(a[-1, 0, 0], bb.c)))
    b.kernel("K2", (d, esqrt(eabs(c.c)) / (a.c - bb.c)))                          # x/0 where a == b
    b.kernel("K3", (e, -(emax(d.c, c[0, 1, 0]) * emin(esqrt(a.c), d[0, 0, -1]))))   # sqrt(<0)
    return b.build()


def special_inputs(desc, seed):
    rng = np.random.default_rng(seed)
    dt = np.float32 if desc.dtype == DT_F32 else np.float64
    specials = np.array([np.nan, np.inf, -np.inf, 0.0, -0.0, 1.0, -1.0, 2.5], dtype=dt)
    out = {}
    for nm, _ in desc.arrays:
        v = rng.uniform(-2, 2, size=desc.padded_shape()).astype(dt)
        m = rng.random(v.shape) < 0.3
        v[m] = specials[rng.integers(0, len(specials), size=int(m.sum()))]
        out[nm] = v
    eq = rng.random(out["a"].shape) < 0.1
    out["b"][eq] = out["a"][eq]                                                     # division by +-0
    return out


@pytest.mark.parametrize("dtype", [DT_F64, DT_F32])
def test_special_values_every_opcode_every_plan(dtype):
    desc = special_program(dtype)
    inputs = special_inputs(desc, 17)
    ref = interp.run(desc, inputs, 2)
    assert any(np.isnan(ref["e"]).ravel()) and any(np.isinf(ref["d"]).ravel())
    plans = En.legal_plans(desc)
    assert len(plans) >= 2
    for plan in plans:
        for tgt in (kf.Target(tile=(16, 4, 0)), kf.Target(tile=(16, 4, 0), pblock=(2, 1), pair_zq=1, canvas_ld=1)):
            got, _ = run_kf(desc, plan, inputs, 2, tgt)
            assert compare_nan(desc, got, ref) == [], (plan, tgt.pblock)


@pytest.mark.parametrize("ghost", [(2, 2, 2), (3, 3, 2)])
def test_ghostwrite_pair_canvas_drops_fills(ghost):
    desc = P.weather(n=(64, 48, 12), ghost=ghost)
    inputs = D.inputs_for(desc, 21)
    ref = interp.run(desc, inputs, 3)
    prog = kf.Program(desc)
    for pb, zq in (((2, 1), 1), ((2, 1), 0), ((1, 1), 1)):
        tgt = kf.Target(tile=(32, 8, 0), pblock=pb, pair_zq=zq, ghostwrite=1, minblocks=-1)
        plan, _ = prog.search(kf.SEARCH_HGGA, tgt, seed=2)      # legal under this launch config (V8)
        got, ex = run_kf(desc, plan, inputs, 3, tgt)
        assert ex.info().fills_per_step == 0
        from .gpu_util import compare
        assert compare(desc, got, ref) == [], (pb, zq)


def test_kf_run_one_call_interface():
    desc = P.weather(n=(48, 40, 12))
    inputs = D.inputs_for(desc, 4)
    ref = interp.run(desc, inputs, 3)
    prog = kf.Program(desc)
    plan = P.weather_hand_plan(desc)
    sb = prog.scratch_bytes(plan)
    assert sb == kf.Exec(prog, plan).scratch_bytes()
    dev = kf.device_arrays(prog, inputs)
    scr = torch.empty(max(sb, 1), dtype=torch.uint8, device="cuda")
    prog.run(plan, dev, scr, 2)
    prog.run([v + 7 for v in plan], dev, scr, 1)     # same canonical plan: the cached executor
    torch.cuda.synchronize()
    from .gpu_util import compare
    assert compare(desc, kf.host_arrays(prog, dev), ref) == []
    with pytest.raises(kf.KfError, match="KF_E_ILLEGAL_PLAN"):
        prog.run([0] * 44, dev, scr, 1)


def test_invalidate_after_frozen_ghost_change():
    """Renamed scratch versions carry copies of the array's FROZEN ghosts; after the caller
    rewrites ghosts under the same pointers, kf_exec_invalidate makes the next run use them."""
    desc = P.tiny(n=(24, 20, 16), flags=PROG_RELAX_ALL)
    inputs = D.uniform(desc, 3)
    prog = kf.Program(desc)
    plan = [0, 0, 0]
    ex = kf.Exec(prog, plan)
    dev = kf.device_arrays(prog, inputs)
    sb = ex.scratch_bytes()
    assert sb > 0
    scr = torch.empty(sb, dtype=torch.uint8, device="cuda")
    ex.run(dev, scr, 1)
    inputs2 = {k: v.copy() for k, v in inputs.items()}
    rng = np.random.default_rng(5)
    for nm in inputs2:
        inside = np.zeros(inputs2[nm].shape, bool)
        inside[2:-2, 2:-2, 2:-2] = True
        inputs2[nm][~inside] = rng.uniform(-3, 3, size=int((~inside).sum())).astype(np.float32)
    for x, (nm, _) in enumerate(desc.arrays):
        dev[x].copy_(torch.from_numpy(prog.to_device_layout(inputs2[nm])))
    ex.invalidate()
    ex.run(dev, scr, 2)
    torch.cuda.synchronize()
    from .gpu_util import compare
    assert compare(desc, kf.host_arrays(prog, dev), interp.run(desc, inputs2, 2)) == []


def _loopback(desc, plan, inputs, nsteps, px, py, target, overlap=True, graph=True):
    parts_np, local = kf.split_domain(desc, inputs, px, py)
    prog = kf.Program(local)
    execs = [kf.Exec(prog, plan, target) for _ in range(px * py)]
    dist = kf.Dist(execs, px, py)
    dist.set_overlap(overlap)
    dist.set_graph(graph)
    dev = [kf.device_arrays(prog, part) for part in parts_np]
    sb = execs[0].scratch_bytes()
    scr = [torch.empty(sb, dtype=torch.uint8, device="cuda") if sb else None for _ in execs]
    dist.run(dev, scr, nsteps)
    torch.cuda.synchronize()
    return kf.gather_domain(desc, [kf.host_arrays(prog, d) for d in dev], px, py, inputs)


def test_dist_periodic_z_with_overlap():
    from .gpu_util import compare
    desc = P.weather(n=(96, 64, 10)).with_(bc=(BC_PERIODIC, BC_PERIODIC, BC_PERIODIC))
    inputs = D.inputs_for(desc, 8)
    ref = interp.run(desc, inputs, 3)
    tgt = kf.Target(tile=(16, 8, 0))
    for plan in (P.weather_hand_plan(desc), list(range(44))):
        got = _loopback(desc, plan, inputs, 3, 2, 2, tgt, overlap=True)
        assert compare(desc, got, ref) == [], plan


@pytest.mark.parametrize("graph", [True, False])
def test_dist_graph_and_eager(graph):
    from .gpu_util import compare
    desc = P.weather(n=(128, 96, 10))
    inputs = D.inputs_for(desc, 12)
    ref = interp.run(desc, inputs, 4)
    tgt = kf.Target(tile=(16, 8, 0), pblock=(2, 1))
    plan = kf.Program(desc).search(kf.SEARCH_HGGA, tgt, seed=1)[0]
    got = _loopback(desc, plan, inputs, 4, 2, 2, tgt, overlap=True, graph=graph)
    assert compare(desc, got, ref) == []


@pytest.mark.parametrize("level", [0, 1, 2])
def test_inline_recompute_levels_bit_exact(level):
    """kf_target.inline_xy (pair canvas): readers recompute in-group values at xy offsets from the
    staged inputs (1), also through recomputed values (2), or read shared-memory copies (0) --
    the same IEEE operations in the same order, so the same bits as the oracle; on the weather
    program (flux -> divergence chains, both periodic seams, ragged tiles) and on random programs."""
    from .gpu_util import compare
    for n, tile in (((64, 48, 12), (32, 8, 0)), ((40, 36, 10), (32, 8, 4)), ((64, 48, 12), (32, 8, 5))):
        desc = P.weather(n=n)     # (z chunks: partial canvas iterations at the interior chunk boundaries)
        inputs = D.inputs_for(desc, 41)
        ref = interp.run(desc, inputs, 2)
        prog = kf.Program(desc)
        tgt = kf.Target(tile=tile, pblock=(2, 1), inline_xy=level, minblocks=-1)
        plan, _ = prog.search(kf.SEARCH_HGGA, tgt, seed=5)
        got, _ = run_kf(desc, plan, inputs, 2, tgt)
        assert compare(desc, got, ref) == [], (n, tile, level)
    for seed in range(4):
        rng = np.random.default_rng(7000 + seed)
        bc = tuple(int(x) for x in rng.integers(0, 2, size=3))
        dtype = DT_F64 if seed % 2 else DT_F32
        desc = P.random_program(7100 + seed, nk=6, na=4, n=(2 * int(rng.integers(8, 16)), 20, 8), dtype=dtype, bc=bc,
                                max_r=1 + seed % 2)
        inputs = D.uniform(desc, seed)
        ref = interp.run(desc, inputs, 2)
        for plan in sorted(En.legal_plans(desc), key=lambda p: len(set(p)))[:3]:
            got, _ = run_kf(desc, plan, inputs, 2, kf.Target(tile=(16, 8, 3), pblock=(2, 1), inline_xy=level))
            assert compare(desc, got, ref) == [], (seed, plan, level)
