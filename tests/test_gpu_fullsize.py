"""Parity at BASELINE full size (config 3: weather 512x512x128 fp64) in the launch configuration
bench.py times (HGGA plan, tile 32x8), checked on sampled windows the oracle computes exactly:
each window is re-run by the oracle on a crop whose margin covers the step's dependency cone
(computed from the kernels' footprints), so the window's values are the exact global result."""
import numpy as np
import pytest

from oracle import interp
from oracle.windows import crop, dependency_radius
from workloads import data as D
from workloads import programs as P

from .gpu_util import bits

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a GPU", allow_module_level=True)

import paper_conf_sc_wahibm14_b200 as kf  # noqa: E402


def test_weather_full_size_sampled_windows():
    desc = P.weather(n=(512, 512, 128))
    inputs = D.weather_inputs(desc, 3)
    prog = kf.Program(desc)
    tgt = kf.Target(tile=(32, 8, 0))
    plan, _ = prog.search(kf.SEARCH_HGGA, tgt, seed=1)
    nsteps = 2
    ex = kf.Exec(prog, plan, tgt)
    dev = kf.device_arrays(prog, inputs)
    sb = ex.scratch_bytes()
    scr = torch.empty(sb, dtype=torch.uint8, device="cuda") if sb else None
    ex.run(dev, scr, nsteps)
    torch.cuda.synchronize()
    got = kf.host_arrays(prog, dev)
    del dev, scr
    M = dependency_radius(desc, nsteps) + 1
    w = 8
    g = desc.ghost
    live = [nm for nm in ("DENS", "MOMX", "MOMY", "MOMZ", "RHOT")]
    for (x0, y0) in ((0, 0), (508, 3), (200, 505), (131, 257)):
        sub, sin = crop(desc, inputs, x0, y0, w, M)
        ref = interp.run(sub, sin, nsteps)
        for nm in live:
            r = ref[nm][g[2]:g[2] + 128, g[1] + M:g[1] + M + w, g[0] + M:g[0] + M + w]
            xs = (np.arange(x0, x0 + w) % 512) + g[0]
            ys = (np.arange(y0, y0 + w) % 512) + g[1]
            gv = got[nm][g[2]:g[2] + 128][:, ys][:, :, xs]
            assert np.array_equal(bits(gv), bits(r)), (nm, x0, y0)


def test_weather_full_size_bench_configuration():
    """The exact configuration of the committed bench line (profiles/bench_timed_config.json,
    refreshed with every committed bench: its plan labels and autotuned per-group launch
    configurations -- canvas pairs, z register queues, unpredicated loads, TMA stages, z chunks,
    ghost writes), at full size, on sampled windows."""
    import json
    import os
    line = json.load(open(os.path.join(os.path.dirname(__file__), "..", "profiles", "bench_timed_config.json")))
    plan = line["plan_labels"]
    tuned = line["per_group_launch_config"]
    gw = line.get("ghostwrite", 0)
    desc = P.weather(n=(512, 512, 128))
    inputs = D.weather_inputs(desc, 3)
    prog = kf.Program(desc)
    import bench
    gt = [kf.Target(**dict(bench.cand_kw({}, c), ghostwrite=gw)) for c in tuned]
    nsteps = 2
    ex = kf.Exec(prog, plan, kf.Target(tile=(32, 8, 64)), group_targets=gt)
    if gw:
        assert ex.info().fills_per_step == 0
    dev = kf.device_arrays(prog, inputs)
    sb = ex.scratch_bytes()
    scr = torch.empty(sb, dtype=torch.uint8, device="cuda") if sb else None
    ex.run(dev, scr, nsteps)
    torch.cuda.synchronize()
    got = kf.host_arrays(prog, dev)
    del dev, scr
    M = dependency_radius(desc, nsteps) + 1
    w = 8
    g = desc.ghost
    for (x0, y0) in ((0, 0), (508, 3), (200, 505), (131, 257), (64, 64), (504, 504)):
        sub, sin = crop(desc, inputs, x0, y0, w, M)
        ref = interp.run(sub, sin, nsteps)
        for nm in ("DENS", "MOMX", "MOMY", "MOMZ", "RHOT"):
            r = ref[nm][g[2]:g[2] + 128, g[1] + M:g[1] + M + w, g[0] + M:g[0] + M + w]
            xs = (np.arange(x0, x0 + w) % 512) + g[0]
            ys = (np.arange(y0, y0 + w) % 512) + g[1]
            gv = got[nm][g[2]:g[2] + 128][:, ys][:, :, xs]
            assert np.array_equal(bits(gv), bits(r)), (nm, x0, y0)
