"""NEXT-4 temporal unrolling (workloads.program.unroll): the description of S timesteps as one step.
Pinned by definition: one step of the unrolled program equals S steps of the original, bit for bit
(the oracle interpreter on both), and the library builds its DAG/legality over the 2*n kernels."""
import numpy as np
import pytest

from oracle import interp
from workloads import data as D
from workloads import programs as P
from workloads.program import unroll


@pytest.mark.parametrize("which", ["tiny", "weather"])
def test_unrolled_step_equals_two_steps(which):
    desc = P.tiny(n=(12, 10, 8)) if which == "tiny" else P.weather(n=(16, 12, 6))
    inputs = D.inputs_for(desc, 4)
    u = unroll(desc, 2)
    assert len(u.kernels) == 2 * len(desc.kernels)
    a = interp.run(desc, inputs, 4)
    b = interp.run(u, inputs, 2)
    for nm in a:
        assert np.array_equal(a[nm].view(np.uint8), b[nm].view(np.uint8)), nm


def test_unrolled_weather_plans_cross_steps():
    kf = pytest.importorskip("paper_conf_sc_wahibm14_b200")
    desc = P.weather(n=(64, 48, 12), ghost=(4, 4, 2))   # cross-step halos need a deeper periodic ghost (V6)
    u = unroll(desc, 2)
    prog = kf.Program(u)
    t = kf.Target(tile=(32, 8, 0))
    plan, b2 = prog.search(kf.SEARCH_HGGA_BYTES, t, seed=1)
    assert prog.validate(plan, t)[0] == 0
    _, b1 = kf.Program(desc).search(kf.SEARCH_HGGA_BYTES, t, seed=1)
    # some group spans the two timesteps, and the unrolled plan moves fewer bytes per timestep
    n = len(desc.kernels)
    assert any(len({k < n for k in range(2 * n) if plan[k] == g}) == 2 for g in set(plan))
    assert b2 / 2 < b1
