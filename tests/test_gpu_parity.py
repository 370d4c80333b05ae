"""GPU parity: the CUDA path (through the C ABI) vs the oracle, element by element.

fp64 bit-exact, fp32 within 2e-6 normwise and in practice bit-exact (north_star).
Sizes span several tiles with ragged tails; full BASELINE sizes are checked on sampled
windows (tests/test_gpu_fullsize.py)."""
import numpy as np
import pytest

from oracle import enum as En
from oracle import interp
from oracle import legality as L
from workloads import data as D
from workloads import programs as P
from workloads.program import BC_FROZEN, BC_PERIODIC, DT_F32, DT_F64, PROG_RELAX_ALL, PROG_RELAX_EXPANDABLE

from .gpu_util import compare, run_kf

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a GPU", allow_module_level=True)

import paper_conf_sc_wahibm14_b200 as kf  # noqa: E402


def test_tiny_config1_all_legal_plans():
    """BASELINE config 1: 32^3 fp32, 4 steps, every legal plan (unfused and {K1,K2}{K3})."""
    desc = P.tiny()
    inputs = D.uniform(desc, 1)
    ref = interp.run(desc, inputs, 4)
    plans = En.legal_plans(desc)
    assert len(plans) == 2
    for plan in plans:
        got, _ = run_kf(desc, plan, inputs, 4)
        assert compare(desc, got, ref) == [], plan


def test_tiny_closed_form_on_gpu():
    desc = P.tiny()
    inputs = D.quadratic(desc)
    got, _ = run_kf(desc, [0, 0, 1], inputs, 1)
    g = desc.ghost
    w = got["w"][g[2] + 1:-g[2] - 1, g[1] + 1:-g[1] - 1, g[0] + 1:-g[0] - 1]
    assert np.all(w == 0.0)                       # L7(L7(quadratic)) = L7(12) = 0 away from the boundary
    assert compare(desc, got, interp.run(desc, inputs, 1)) == []


@pytest.mark.parametrize("tile", [(32, 16, 0), (16, 8, 0), (32, 16, 7), (8, 8, 5)])
@pytest.mark.parametrize("zunroll", [1, 2, 3])
@pytest.mark.parametrize("ringunroll", [0, 1])
def test_tiny_ragged_tiles_and_z_chunks(tile, zunroll, ringunroll):
    desc = P.tiny(n=(37, 21, 19))
    inputs = D.uniform(desc, 2)
    ref = interp.run(desc, inputs, 3)
    got, _ = run_kf(desc, [0, 0, 1], inputs, 3, kf.Target(tile=tile, zunroll=zunroll, ringunroll=ringunroll))
    assert compare(desc, got, ref) == []


def test_fig3_all_20_legal_plans_fp64():
    """Fig. 3 kernels in fp64: every legal plan, including the paper's X,Y, bit-exact."""
    desc = P.fig3(n=(40, 24, 10))
    inputs = D.inputs_for(desc, 3)
    ref = interp.run(desc, inputs, 1)
    plans = En.legal_plans(desc)
    assert len(plans) == 20
    for plan in plans:
        got, _ = run_kf(desc, plan, inputs, 1)
        assert compare(desc, got, ref) == [], plan


@pytest.mark.parametrize("seed", range(16))
def test_random_programs_random_legal_plans(seed):
    rng = np.random.default_rng(1000 + seed)
    bc = tuple(int(x) for x in rng.integers(0, 2, size=3))
    flags = [0, PROG_RELAX_EXPANDABLE, PROG_RELAX_ALL][seed % 3]
    dtype = DT_F32 if seed % 2 else DT_F64
    n = tuple(int(x) for x in rng.integers(9, 40, size=3))
    desc = P.random_program(2000 + seed, nk=5, na=4, n=n, dtype=dtype, bc=bc, flags=flags, max_r=1 + seed % 2)
    inputs = D.uniform(desc, seed)
    nsteps = 1 + seed % 3
    ref = interp.run(desc, inputs, nsteps)
    legal = En.legal_plans(desc)
    pick = [legal[i] for i in sorted(set(rng.integers(0, len(legal), size=4).tolist()))]
    tile = [(32, 16, 0), (16, 16, 0), (8, 4, 6), (32, 8, 11)][seed % 4]
    zu = [1, 2, 3][seed % 3]
    pb = [(1, 1), (2, 1), (2, 2), (1, 3)][seed % 4]
    ru = seed % 2
    gw = (seed // 2) % 2
    ran = 0
    for plan in pick:
        t = kf.Target(tile=tile, zunroll=zu, pblock=pb, threads=64, ringunroll=ru, ghostwrite=gw)
        if kf.Program(desc).validate(plan, t)[0] in (7, 8):   # resource model rejects this launch config
            with pytest.raises(kf.KfError, match="KF_E_ILLEGAL_PLAN"):
                kf.Exec(kf.Program(desc), plan, t)
            t = kf.Target(tile=tile, zunroll=1, pblock=(1, 1), ringunroll=ru, ghostwrite=gw)
        got, _ = run_kf(desc, plan, inputs, nsteps, t)
        assert compare(desc, got, ref) == [], (plan, tile)
        ran += 1
    assert ran >= 1


def test_weather_small_fp64_plans():
    """Config 3 program at a small size: unfused, the hand plan and the searched plan, 2 steps."""
    from workloads.programs import weather_hand_plan
    desc = P.weather(n=(48, 40, 12))
    inputs = D.inputs_for(desc, 3)
    ref = interp.run(desc, inputs, 2)
    plan_g, _ = kf.Program(desc).search(kf.SEARCH_GREEDY, kf.Target(tile=(32, 8, 0), zunroll=2))
    for plan in (list(range(44)), weather_hand_plan(desc), plan_g):
        for zu, ru, gw in ((1, 0, 1), (2, 0, 0), (1, 1, 1)):
            got, _ = run_kf(desc, plan, inputs, 2, kf.Target(tile=(32, 8, 0), zunroll=zu, ringunroll=ru, ghostwrite=gw))
            assert compare(desc, got, ref) == [], (plan, zu, ru)


def test_graph_and_eager_agree_and_odd_even_steps():
    desc = P.weather(n=(32, 32, 8))
    inputs = D.inputs_for(desc, 5)
    plan, _ = kf.Program(desc).search(kf.SEARCH_GREEDY)
    for nsteps in (1, 2, 3):
        ref = interp.run(desc, inputs, nsteps)
        for graph in (True, False):
            got, _ = run_kf(desc, plan, inputs, nsteps, graph=graph)
            assert compare(desc, got, ref) == [], (nsteps, graph)


def test_registers_within_model_and_no_spills():
    """V8's register model must bound ptxas (R20); no local-memory spills."""
    desc = P.weather(n=(64, 64, 16))
    plan, _ = kf.Program(desc).search(kf.SEARCH_GREEDY)
    _, ex = run_kf(desc, plan, D.inputs_for(desc, 1), 1)
    per, _, _ = kf.Program(desc).project(plan)
    for g in range(ex.info().n_groups):
        gi = ex.group_info(g)
        assert gi.local_bytes == 0, gi.name
        assert gi.regs <= per[g].regs_est, (gi.name, gi.regs, per[g].regs_est)


def test_run_host_path():
    desc = P.tiny(n=(24, 20, 16))
    inputs = D.uniform(desc, 9)
    prog = kf.Program(desc)
    ex = kf.Exec(prog, [0, 0, 1])
    host = [torch.from_numpy(prog.to_device_layout(inputs[nm])).pin_memory() for nm, _ in desc.arrays]
    h2d, d2h = ex.run_host([t.data_ptr() for t in host], 3)
    got = {nm: prog.from_device_layout(t.numpy()) for (nm, _), t in zip(desc.arrays, host)}
    assert compare(desc, got, interp.run(desc, inputs, 3)) == []
    assert h2d > 0 and d2h > 0


def test_per_group_launch_configs():
    """kf_exec_create_ex: every group with its own tile / stages / zunroll, bit-exact."""
    from workloads.programs import weather_hand_plan
    desc = P.weather(n=(40, 36, 10))
    inputs = D.inputs_for(desc, 7)
    ref = interp.run(desc, inputs, 2)
    plan = weather_hand_plan(desc)
    m = max(plan) + 1
    cfgs = [((64, 4, 0), 2, 1, (1, 1), 256), ((32, 8, 0), 2, 2, (2, 1), 256), ((16, 8, 3), 3, 1, (1, 2), 64),
            ((32, 4, 0), 2, 3, (1, 1), 128), ((64, 8, 0), 2, 1, (2, 2), 256)]
    tg = [kf.Target(tile=cfgs[g % 5][0], stages=cfgs[g % 5][1], zunroll=cfgs[g % 5][2], pblock=cfgs[g % 5][3],
                    threads=cfgs[g % 5][4]) for g in range(m)]
    prog = kf.Program(desc)
    ex = kf.Exec(prog, plan, group_targets=tg)
    dev = kf.device_arrays(prog, inputs)
    sb = ex.scratch_bytes()
    scratch = torch.empty(sb, dtype=torch.uint8, device="cuda") if sb else None
    ex.run(dev, scratch, 2)
    torch.cuda.synchronize()
    assert compare(desc, kf.host_arrays(prog, dev), ref) == []


def test_suite_config2_every_legal_plan():
    """BASELINE config 2 shape (10 kernels / 8 arrays, mixed 7/13/27-point fp32 stencils, periodic
    xy): every legal plan of a generated program runs bit-exactly (grid reduced to 40x32x12)."""
    desc = P.gen_suite(seed=1, n=(40, 32, 12))
    inputs = D.uniform(desc, 2)
    ref = interp.run(desc, inputs, 3)
    prog = kf.Program(desc)
    legal = En.legal_plans(desc) if False else None
    n = prog.count_legal()
    assert n == 188
    # enumerate through the oracle's restricted-growth strings, keeping the library-legal ones
    tgt = kf.Target(tile=(16, 8, 0))
    checked = 0
    for plan in En.restricted_growth(10):
        if prog.validate(plan, tgt)[0] != 0:
            continue
        got, _ = run_kf(desc, plan, inputs, 3, tgt)
        assert compare(desc, got, ref) == [], plan
        checked += 1
    assert checked == prog.count_legal(tgt)


@pytest.mark.parametrize("tile", [(32, 8, 0), (16, 8, 0)])
def test_stress_config5_radius4_plans(tile):
    """BASELINE config 5 shape: radius-4 (25-point) fp64 stencils L25(L25(f)) + update, RELAX_ALL,
    ghost 8, periodic xy; every legal plan (the fully fused group sits near the SMEM limit)."""
    desc = P.stress(m=2, n=(40, 36, 20))
    inputs = D.uniform(desc, 5)
    ref = interp.run(desc, inputs, 2)
    prog = kf.Program(desc)
    tgt = kf.Target(tile=tile)
    n = 0
    for plan in En.restricted_growth(6):
        if prog.validate(plan, tgt)[0] != 0:
            continue
        got, _ = run_kf(desc, plan, inputs, 2, tgt)
        assert compare(desc, got, ref) == [], plan
        n += 1
    assert n == prog.count_legal(tgt) >= 4


@pytest.mark.parametrize("seed", range(8))
def test_canvas_paths_random_programs(seed, monkeypatch):
    """Canvas fast iterations (one canvas point per thread: register forwarding, cross-kernel load
    CSE) under every codegen knob: delay skew, z-queue carries (KF_CQ), register cap, z-unroll,
    unpredicated / predicated shared loads (canvas_ld)."""
    rng = np.random.default_rng(3000 + seed)
    bc = tuple(int(x) for x in rng.integers(0, 2, size=3))
    flags = [0, PROG_RELAX_EXPANDABLE, PROG_RELAX_ALL][seed % 3]
    dtype = DT_F64 if seed % 2 else DT_F32
    n = tuple(int(x) for x in rng.integers(12, 40, size=3))
    desc = P.random_program(4000 + seed, nk=6, na=4, n=n, dtype=dtype, bc=bc, flags=flags, max_r=1 + seed % 2)
    inputs = D.uniform(desc, seed)
    nsteps = 1 + seed % 2
    ref = interp.run(desc, inputs, nsteps)
    legal = En.legal_plans(desc)
    # the plans with the largest groups exercise forwarding the most
    pick = sorted(legal, key=lambda p: len(set(p)))[:3]
    if seed % 2:
        monkeypatch.setenv("KF_CQ", "1")
    tile = [(16, 8, 0), (8, 8, 7), (32, 4, 0), (16, 4, 9)][seed % 4]
    for plan in pick:
        for skew, mb, zu, cl, pb in ((0, 0, 1, 1, 1), (0, 0, 1, 0, 1), (1, -1, 1, 1, 1), (seed % 2, 0, 2, seed % 2, 1),
                                     (0, 0, 1, 1, 2), (0, -1, 1, 0, 2)):
            t = kf.Target(tile=tile, skew=skew, minblocks=mb, zunroll=zu, canvas_ld=cl, pblock=(pb, 1))
            got, _ = run_kf(desc, plan, inputs, nsteps, t)
            assert compare(desc, got, ref) == [], (plan, tile, skew, mb, zu, cl, pb)


@pytest.mark.parametrize("seed", range(6))
def test_canvas_pairs_random_programs(seed):
    """Pair mode of the canvas (pblock 2x1: two x-adjacent points per thread, 16-byte vector shared
    loads/stores and live-out stores) on random programs with even nx, every boundary condition mix,
    both dtypes, predicated and unpredicated loads, with and without z-column register queues."""
    rng = np.random.default_rng(5000 + seed)
    bc = tuple(int(x) for x in rng.integers(0, 2, size=3))
    flags = [0, PROG_RELAX_EXPANDABLE, PROG_RELAX_ALL][seed % 3]
    dtype = DT_F64 if seed % 2 else DT_F32
    n = (2 * int(rng.integers(8, 20)), int(rng.integers(10, 30)), int(rng.integers(6, 14)))
    desc = P.random_program(6000 + seed, nk=6, na=4, n=n, dtype=dtype, bc=bc, flags=flags, max_r=1 + seed % 2)
    inputs = D.uniform(desc, seed)
    ref = interp.run(desc, inputs, 2)
    legal = En.legal_plans(desc)
    pick = sorted(legal, key=lambda p: len(set(p)))[:3]
    tile = [(16, 8, 0), (8, 8, 5), (32, 4, 0)][seed % 3]
    for plan in pick:
        for cl, zq in ((0, 1), (1, 1), (1, 0)):
            got, _ = run_kf(desc, plan, inputs, 2, kf.Target(tile=tile, pblock=(2, 1), canvas_ld=cl, pair_zq=zq))
            assert compare(desc, got, ref) == [], (plan, tile, cl, zq)


@pytest.mark.parametrize("cq", [0, 1])
def test_canvas_weather_knobs(cq, monkeypatch):
    """Weather program (config 3 shape, small grid): the bench's plan family with the canvas knobs."""
    if cq:
        monkeypatch.setenv("KF_CQ", "1")
    desc = P.weather(n=(64, 48, 12))
    inputs = D.inputs_for(desc, 4)
    ref = interp.run(desc, inputs, 2)
    prog = kf.Program(desc)
    tgt = kf.Target(tile=(32, 8, 0))
    # plans searched for single points and for pairs (V8 differs: the pair canvas holds more values)
    plans = [prog.search(kf.SEARCH_HGGA, tgt, seed=s)[0] for s in (1, 2)] + \
        [prog.search(kf.SEARCH_HGGA, kf.Target(tile=(32, 8, 0), pblock=(2, 1)), seed=s)[0] for s in (1, 2)]
    for plan in plans:
        for kw in (dict(), dict(canvas_ld=0), dict(pblock=(2, 1)), dict(pblock=(2, 1), canvas_ld=0),
                   dict(pblock=(2, 1), pair_zq=0), dict(skew=1),
                   dict(minblocks=-1, ringunroll=1), dict(tile=(32, 8, 5))):
            t = kf.Target(**dict(dict(tile=(32, 8, 0)), **kw))
            if prog.validate(plan, t)[0] != 0:   # e.g. V7: skew / ring unrolling need more SMEM; V8
                continue
            got, _ = run_kf(desc, plan, inputs, 2, t)
            assert compare(desc, got, ref) == [], (plan, kw)


@pytest.mark.parametrize("nk,load", [(30, 4), (40, 8), (24, 12)])
def test_suite_sweep_programs_parity(nk, load):
    """NEXT-3 test-suite programs (Table V thread loads 4/8/12): the HGGA plans vs the oracle."""
    desc = P.gen_suite(n_kernels=nk, n_arrays=2 * nk, seed=1, n=(40, 32, 12), load=load, max_tries=2000)
    inputs = D.uniform(desc, 7)
    ref = interp.run(desc, inputs, 2)
    prog = kf.Program(desc)
    tgt = kf.Target(tile=(32, 8, 0))
    for method in (kf.SEARCH_HGGA, kf.SEARCH_HGGA_BYTES):
        plan, _ = prog.search(method, tgt, seed=1)
        got, _ = run_kf(desc, plan, inputs, 2, tgt)
        assert compare(desc, got, ref) == [], (method, plan)
