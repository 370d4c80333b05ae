"""A/B of per-group launch configurations on one fixed plan, alternating variants (ABAB...) to
cancel drift (power/clock state).  Prints one JSON line per variant with the median over rounds of
the step time and of every group's time.

  python tools/round2/abt.py '<json spec>'
  spec = {"workload": "weather", "plan": [...labels], "tuned": [[tile, stages, zunroll, ringunroll,
          minblocks, canvas_ld, pblock_x, pair_zq], ...], "variants": [{"name": .., "ghostwrite": 0|1,
          "override": {group: [...config]}, "env": {..},
          "target": {kf_target field: value}}], "rounds": 5, "steps": 10}
"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_sc_wahibm14_b200 as kf  # noqa: E402


def main():
    spec = json.loads(sys.argv[1])
    torch.cuda.set_device(0)
    wl = bench.Workload(spec.get("workload", "weather"), 1)
    prog = kf.Program(wl.desc)
    dev, _ = wl.inputs(prog, 0)
    plan = spec["plan"]
    steps = spec.get("steps", 10)
    runs = []
    for v in spec["variants"]:
        plan = v.get("plan", spec["plan"])
        tuned = [list(c) for c in v.get("tuned", spec["tuned"])]
        for g, c in v.get("override", {}).items():
            tuned[int(g)] = c
        old = {}
        for k, val in v.get("env", {}).items():
            old[k] = os.environ.get(k)
            os.environ[k] = str(val)
        base = dict(wl.tkw, ghostwrite=v.get("ghostwrite", 1))
        base.update(v.get("target", {}))   # e.g. {"wrapload": 1}
        gt = [kf.Target(**bench.cand_kw(base, c)) for c in tuned]
        ex = kf.Exec(prog, plan, gt[0], group_targets=gt)
        for k, o in old.items():
            if o is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = o
        sb = ex.scratch_bytes()
        scr = torch.empty(sb, dtype=torch.uint8, device="cuda") if sb else None
        if v.get("dist"):   # loopback kf_dist over one part: periodic fills overlapped with interior tiles
            d = kf.Dist([ex], 1, 1)
            d.set_overlap(True)
            runner = type("R", (), {})()
            runner.ex = ex
            runner.run = (lambda d_: (lambda dev_, scr_, n: d_.run([dev_], [scr_], n)))(d)
            runner.d = d
        else:
            runner = ex
        runs.append((v, runner, scr, [], []))
    for _ in range(spec.get("rounds", 5)):
        for v, ex, scr, st, gt_ in runs:
            ex.run(dev, scr, 2)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            ex.run(dev, scr, steps)
            e1.record()
            torch.cuda.synchronize()
            st.append(e0.elapsed_time(e1) / steps)
            ex.ex.set_profiling(True) if hasattr(ex, "d") else ex.set_profiling(True)
            ex.run(dev, scr, steps)
            torch.cuda.synchronize()
            e_ = ex.ex if hasattr(ex, "d") else ex
            gms, _ = e_.group_times()
            e_.set_profiling(False)
            gt_.append([g / steps for g in gms])
    for v, ex, scr, st, gt_ in runs:
        med = [statistics.median(x) for x in zip(*gt_)]
        ex = ex.ex if hasattr(ex, "d") else ex
        gi = [ex.group_info(g) for g in range(ex.info().n_groups)]
        print(json.dumps({"variant": v.get("name", v), "ms_per_step": round(statistics.median(st), 4),
                          "ms_all": [round(x, 4) for x in st], "fills_per_step": ex.info().fills_per_step,
                          "groups": [(g.name.decode(), round(t, 4), g.regs, g.smem_bytes, g.threads) for g, t in zip(gi, med)]}),
              flush=True)


if __name__ == "__main__":
    main()
