"""Hardware pin of the resource model (V7 / V8, reading R20): for every group of
every bench autotune candidate on configs 2, 3 and 5 at full size, the loaded sm_100a kernel

* launches with exactly the model's dynamic shared memory (V7: smem_bytes == kf_project's),
* uses at most R_est registers (V8: CU_FUNC_ATTRIBUTE_NUM_REGS <= regs_est; R_est is the kernel's
  __maxnreg__ budget), and
* does not spill (CU_FUNC_ATTRIBUTE_LOCAL_SIZE_BYTES == 0) -- i.e. the model's budget is enough.

Candidates V8 rejects (R_est > 255) are counted and must be rejected by kf_plan_validate too."""
import json
import os
from concurrent.futures import ThreadPoolExecutor

import pytest

from workloads import programs as P

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a GPU", allow_module_level=True)

import bench  # noqa: E402
import paper_conf_sc_wahibm14_b200 as kf  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _plans(cfg):
    if cfg == 3:
        desc = P.weather(n=(512, 512, 128))
        prog = kf.Program(desc)
        base = dict(tile=(32, 8, 64))
        t = kf.Target(**base)
        plans = [json.load(open(os.path.join(ROOT, "profiles", "bench_timed_config.json")))["plan_labels"],
                 P.weather_hand_plan(desc)] + [prog.search(kf.SEARCH_HGGA, t, seed=s)[0] for s in (1, 3)]
    elif cfg == 2:
        desc = P.gen_suite(seed=0)
        prog = kf.Program(desc)
        base = dict(tile=(32, 8, 0))
        legal = prog.legal_plans(kf.Target(**base))
        plans = [prog.search(kf.SEARCH_BRUTE_TIME, kf.Target(**base))[0]] + legal[::max(1, len(legal) // 8)]
    else:
        desc = P.stress(m=2, n=(768, 768, 768))
        prog = kf.Program(desc)
        base = dict(tile=(32, 8, 0), max_halo=16)
        nk = len(desc.kernels)
        half = [k * 2 // nk for k in range(nk)]      # the two fields' chains fused per field
        plans = [prog.search(kf.SEARCH_BRUTE_TIME, kf.Target(**base))[0], list(range(nk)), half]
    # only plans legal under the base configuration (V1-V8); the candidates then vary V7/V8 only
    plans = [pl for pl in plans if prog.validate(pl, kf.Target(**base))[0] == 0]
    return prog, base, plans


@pytest.mark.parametrize("cfg", [3, 2, 5])
def test_resource_model_bounds_loaded_kernels(cfg):
    torch.cuda.set_device(0)
    prog, base, plans = _plans(cfg)
    jobs = []
    for plan in plans:
        for cand in bench.AUTOTUNE_CANDIDATES:
            kw = bench.cand_kw(base, cand)
            kw["ghostwrite"] = 0
            jobs.append((plan, kw))

    def make(job):
        plan, kw = job
        t = kf.Target(**kw)
        v = prog.validate(plan, t)
        if v[0] != 0:
            return (job, v, None)
        return (job, v, kf.Exec(prog, plan, t))

    with ThreadPoolExecutor(max_workers=8) as pool:
        made = list(pool.map(make, jobs))
    checked = rejected = 0
    bad = []
    for (plan, kw), v, ex in made:
        per, _, _ = prog.project(plan, kf.Target(**kw))
        if ex is None:
            # only V7/V8 (launch-configuration dependent) may reject a plan the search produced
            assert v[0] in (7, 8), (plan, kw, v)
            rejected += 1
            continue
        ex.load()
        for g in range(ex.info().n_groups):
            gi = ex.group_info(g)
            ok = gi.smem_bytes == per[g].smem_bytes and gi.regs <= per[g].regs_est and gi.local_bytes == 0
            if not ok:
                bad.append((gi.name.decode(), kw["tile"], kw["pblock"], kw["pair_zq"], kw["minblocks"], gi.smem_bytes,
                            per[g].smem_bytes, gi.regs, per[g].regs_est, gi.local_bytes))
            checked += 1
        del ex
    assert not bad, bad[:10]
    assert checked >= 20, (checked, rejected)
