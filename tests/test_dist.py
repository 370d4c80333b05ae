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


def _gloo_strip_worker(rank, world, port, q, axis):
    """Two real processes exchange their halo strips over gloo using kf_dist's strip geometry
    (kf_dist_strips of the LOCAL program, in the kf device layout), as the NCCL transport does:
    pack send_lo/send_hi, send to the low/high neighbour, receive into recv_hi/recv_lo."""
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_sc_wahibm14_b200 as kf
    desc = P.weather(n=(32, 24, 6))
    arrs = D.inputs_for(desc, 5)
    px, py = (world, 1) if axis == 0 else (1, world)
    parts, local = kf.split_domain(desc, arrs, px, py)
    prog = kf.Program(local)
    L_ = prog.layout()
    flat = prog.to_device_layout(parts[rank]["DENS"]).copy()
    flat[:] = np.where(np.isfinite(flat), flat, 0)
    if axis == 1:   # x is not decomposed: local x wrap first (the y strips carry the x ghosts = corners)
        v = flat.reshape(-1, L_.rows, L_.pitch)
        g0 = local.ghost[0]
        v[:, :, L_.xoff - g0:L_.xoff] = v[:, :, L_.xoff + local.n[0] - g0:L_.xoff + local.n[0]]
        v[:, :, L_.xoff + local.n[0]:L_.xoff + local.n[0] + g0] = v[:, :, L_.xoff:L_.xoff + g0]
    boxes = prog.dist_strips(axis)

    def view(b):
        off, w, h, d = b
        return np.lib.stride_tricks.as_strided(flat[off:], shape=(d, h, w),
                                               strides=(L_.plane * 8, L_.pitch * 8, 8))
    lo, hi, dn, up = kf.dist_neighbors(px, py, rank)
    nlo, nhi = (lo, hi) if axis == 0 else (dn, up)
    s_lo = torch.from_numpy(np.ascontiguousarray(view(boxes[0])))
    s_hi = torch.from_numpy(np.ascontiguousarray(view(boxes[1])))
    r_lo, r_hi = torch.empty_like(s_lo), torch.empty_like(s_hi)
    reqs = [dist.isend(s_lo, nlo, tag=0), dist.isend(s_hi, nhi, tag=1),
            dist.irecv(r_hi, nhi, tag=0), dist.irecv(r_lo, nlo, tag=1)]
    for r_ in reqs:
        r_.wait()
    view(boxes[2])[...] = r_lo.numpy()
    view(boxes[3])[...] = r_hi.numpy()
    got = prog.from_device_layout(flat)
    dist.destroy_process_group()
    q.put((rank, got))


@pytest.mark.parametrize("axis", [0, 1])
def test_gloo_two_ranks_exchange_kf_strips(axis):
    """Both ranks' ghost layers after an exchange through kf_dist_strips' boxes equal the global
    field's periodic neighbours (interior, ghosts of the decomposed axis, corners on y)."""
    import multiprocessing as mp
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_gloo_strip_worker, args=(r, 2, port, q, axis)) for r in range(2)]
    for p_ in procs:
        p_.start()
    res = dict(q.get(timeout=180) for _ in procs)
    for p_ in procs:
        p_.join(60)
    desc = P.weather(n=(32, 24, 6))
    a = D.inputs_for(desc, 5)["DENS"]
    gx, gy, gz = desc.ghost
    nx, ny, nz = desc.n
    for r in range(2):
        got = res[r]
        lx, ly = (16, 24) if axis == 0 else (32, 12)
        ox, oy = (16 * r, 0) if axis == 0 else (0, 12 * r)
        # x: interior rows, interior + exchanged x ghost columns; y: whole padded rows (x ghosts by
        # the local wrap = corners) of the interior + exchanged y ghost rows
        ys = np.arange(-gy, ly + gy) if axis == 1 else np.arange(0, ly)
        for j in ys:
            for i in np.arange(-gx, lx + gx):
                gi, gj = (ox + i) % nx, (oy + j) % ny
                assert np.array_equal(got[gz:gz + nz, gy + j, gx + i], a[gz:gz + nz, gy + gj, gx + gi]), (r, i, j)


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
    ran = 0
    for plan in plans:
        for t in (tgt, kf.Target(tile=(16, 8, 0), pblock=(2, 1))):   # single points and canvas pairs
            parts_np, local = kf.split_domain(desc, inputs, 2, 2)
            if kf.Program(local).validate(plan, t)[0] != 0:   # V8: the pair canvas holds more values
                continue
            ran += 1
            got = _run_loopback(desc, plan, inputs, 3, 2, 2, t, overlap=overlap)
            assert compare(desc, got, ref) == [], (overlap, plan, t.pblock)
    assert ran >= 3
