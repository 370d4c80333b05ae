"""Row a11 (multi-GPU domain decomposition).

CPU (gloo, world_size 2): the host logic -- process-grid neighbours, domain split/gather
round trip and the bytes a rank would send -- exercised by two real processes.
GPU (loopback transport, one device): the decomposed run equals the single-domain oracle
bit for bit (the halo exchange replaces the periodic wrap)."""
import os

import numpy as np
import pytest

from oracle import interp
from workloads import data as D
from workloads import programs as P
from workloads.program import BC_FROZEN, BC_PERIODIC, DT_F32, DT_F64, PROG_RELAX_ALL

from .gpu_util import compare


def test_neighbors_periodic_grid():
    kf = pytest.importorskip("paper_conf_sc_wahibm14_b200")
    assert kf.dist_neighbors(4, 2, 0) == [3, 1, 4, 4]
    assert kf.dist_neighbors(4, 2, 5) == [4, 6, 1, 1]
    assert kf.dist_neighbors(1, 1, 0) == [0, 0, 0, 0]
    for px, py in ((2, 1), (2, 2), (4, 2), (3, 3)):
        for r in range(px * py):
            lo, hi, dn, up = kf.dist_neighbors(px, py, r)
            assert kf.dist_neighbors(px, py, lo)[1] == r and kf.dist_neighbors(px, py, hi)[0] == r
            assert kf.dist_neighbors(px, py, dn)[3] == r and kf.dist_neighbors(px, py, up)[2] == r


def test_split_gather_roundtrip():
    kf = pytest.importorskip("paper_conf_sc_wahibm14_b200")
    desc = P.weather(n=(24, 16, 6))
    arrs = D.inputs_for(desc, 1)
    parts, local = kf.split_domain(desc, arrs, 3, 2)
    assert local.n == (8, 8, 6) and len(parts) == 6
    back = kf.gather_domain(desc, parts, 3, 2, {k: np.zeros_like(v) for k, v in arrs.items()})
    g = desc.ghost
    for nm in arrs:
        assert np.array_equal(back[nm][g[2]:-g[2], g[1]:-g[1], g[0]:-g[0]], arrs[nm][g[2]:-g[2], g[1]:-g[1], g[0]:-g[0]])


def _gloo_worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_sc_wahibm14_b200 as kf
    desc = P.weather(n=(32, 16, 6))
    arrs = D.inputs_for(desc, 5)                   # same seed on every rank = the global state
    parts, local = kf.split_domain(desc, arrs, world, 1)
    mine = parts[rank]
    lo, hi, _, _ = kf.dist_neighbors(world, 1, rank)
    g = desc.ghost[0]
    # what this rank sends to its low neighbour (its first g interior columns), checksum gathered
    strip = mine["DENS"][:, :, g:2 * g]
    t = torch.tensor([float(strip.sum()), float(lo), float(hi)], dtype=torch.float64)
    out = [torch.zeros(3, dtype=torch.float64) for _ in range(world)]
    dist.all_gather(out, t)
    dist.destroy_process_group()
    q.put((rank, [o.tolist() for o in out]))


def test_gloo_two_ranks_host_logic():
    import multiprocessing as mp
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_gloo_worker, args=(r, 2, port, q)) for r in range(2)]
    for p_ in procs:
        p_.start()
    res = dict(q.get(timeout=120) for _ in procs)
    for p_ in procs:
        p_.join(60)
    desc = P.weather(n=(32, 16, 6))
    arrs = D.inputs_for(desc, 5)
    g = desc.ghost[0]
    # rank r's first interior columns are global interior columns [16 r, 16 r + g)
    for r in range(2):
        expect = arrs["DENS"][:, :, g + 16 * r:g + 16 * r + g].sum()
        assert res[0][r][0] == pytest.approx(float(expect), rel=0, abs=0)
        assert res[0][r][1:] == [float(1 - r), float(1 - r)]   # in a 2-rank ring both neighbours are the other rank
    assert res[0] == res[1]


# ----------------------------------------------------------------------------------- GPU
def _run_loopback(desc, plan, inputs, nsteps, px, py, target=None, overlap=True):
    import torch
    import paper_conf_sc_wahibm14_b200 as kf
    parts_np, local = kf.split_domain(desc, inputs, px, py)
    prog = kf.Program(local)
    execs = [kf.Exec(prog, plan, target) for _ in range(px * py)]
    dist = kf.Dist(execs, px, py)
    dist.set_overlap(overlap)
    dev = [kf.device_arrays(prog, part) for part in parts_np]
    sb = execs[0].scratch_bytes()
    scr = [torch.empty(sb, dtype=torch.uint8, device="cuda") if sb else None for _ in execs]
    dist.run(dev, scr, nsteps)
    torch.cuda.synchronize()
    got_parts = [kf.host_arrays(prog, d) for d in dev]
    return kf.gather_domain(desc, got_parts, px, py, inputs)


@pytest.mark.gpu
@pytest.mark.parametrize("px,py", [(2, 1), (1, 3), (2, 2), (4, 2)])
def test_loopback_weather_equals_single_domain(px, py):
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    import paper_conf_sc_wahibm14_b200 as kf
    desc = P.weather(n=(48, 36, 10))
    inputs = D.inputs_for(desc, 11)
    ref = interp.run(desc, inputs, 3)
    for plan in (P.weather_hand_plan(desc), list(range(44))):
        got = _run_loopback(desc, plan, inputs, 3, px, py, kf.Target(tile=(16, 8, 0)))
        assert compare(desc, got, ref) == [], (px, py, plan)


@pytest.mark.gpu
def test_loopback_random_periodic_programs():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    import paper_conf_sc_wahibm14_b200 as kf
    from oracle import enum as En
    for seed in range(4):
        dt = DT_F32 if seed % 2 else DT_F64
        desc = P.random_program(300 + seed, nk=4, na=4, n=(24, 18, 7), dtype=dt,
                                bc=(BC_PERIODIC, BC_PERIODIC, BC_FROZEN), flags=PROG_RELAX_ALL if seed >= 2 else 0,
                                max_r=2)
        inputs = D.uniform(desc, seed)
        ref = interp.run(desc, inputs, 2)
        legal = En.legal_plans(desc)
        for plan in (legal[0], legal[-1]):
            got = _run_loopback(desc, plan, inputs, 2, 2, 3, kf.Target(tile=(8, 4, 0)))
            assert compare(desc, got, ref) == [], (seed, plan)


@pytest.mark.gpu
@pytest.mark.parametrize("overlap", [True, False])
def test_loopback_overlap_interior_boundary_split(overlap):
    """Exchange / interior-compute overlap: local sub-domains large enough that every
    group splits into interior tiles (launched while the exchanges run on the second stream) and
    boundary tiles (after them); bit-exact with the oracle with and without the overlap."""
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    import paper_conf_sc_wahibm14_b200 as kf
    desc = P.weather(n=(128, 96, 10))
    inputs = D.inputs_for(desc, 12)
    ref = interp.run(desc, inputs, 3)
    tgt = kf.Target(tile=(16, 8, 0))
    plans = [P.weather_hand_plan(desc), kf.Program(desc).search(kf.SEARCH_HGGA, tgt, seed=1)[0]]
    for plan in plans:
        for t in (tgt, kf.Target(tile=(16, 8, 0), pblock=(2, 1))):   # single points and canvas pairs
            got = _run_loopback(desc, plan, inputs, 3, 2, 2, t, overlap=overlap)
            assert compare(desc, got, ref) == [], (overlap, plan, t.pblock)
