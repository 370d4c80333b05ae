"""A/B measurement of launch configurations / codegen knobs on one fixed weather plan.

  python tools/ab.py '<variants json>' [plan: hgga|hand|unfused|<labels json>]

Each variant is {"tile": [..], "stages": S, "zunroll": U, "pblock": [bx, by], "ringunroll": R,
"env": {"KF_ZQ_MAX": "64", ...}}; every group of the plan is compiled with it and timed with
per-group CUDA events (10 steps after 3 warm-up steps).  Prints one JSON line per variant.
"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_wahibm14_b200 as kf
from workloads import programs as P, data as D

HGGA = [0, 0, 0, 1, 1, 1, 1, 1, 1, 2, 2, 2, 2, 2, 2, 0, 2, 0, 0, 0, 0, 1, 1, 1, 1, 2, 2, 3, 2, 2, 4, 4, 3, 5, 5, 4,
        4, 3, 5, 3, 4, 4, 3, 5]


def main():
    variants = json.loads(sys.argv[1])
    which = sys.argv[2] if len(sys.argv) > 2 else "hgga"
    wl = sys.argv[3] if len(sys.argv) > 3 else "weather"
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import bench
    w = bench.Workload(wl, 1)
    desc, tkw = w.desc, dict(w.tkw)
    prog = kf.Program(desc)
    if which == "best":
        plan = bench.choose_plan(prog, kf.Target(**tkw), "best")[0]
    elif wl == "weather":
        plan = {"hgga": HGGA, "hand": P.weather_hand_plan(desc), "unfused": list(range(44))}.get(which) or json.loads(which)
    else:
        plan = list(range(prog.nk)) if which == "unfused" else json.loads(which)
    dev, _ = w.inputs(prog, 0)
    print(json.dumps({"workload": wl, "plan": plan}), flush=True)
    steps = int(os.environ.get("AB_STEPS", "10"))
    for v in variants:
        saved = {}
        for k, val in v.get("env", {}).items():
            saved[k] = os.environ.get(k)
            os.environ[k] = str(val)
        kw = {k: (tuple(x) if isinstance(x, list) else x) for k, x in v.items() if k != "env"}
        try:
            ex = kf.Exec(prog, plan, kf.Target(**kw))
        except Exception as e:
            print(json.dumps({"variant": v, "error": str(e)[:300]}), flush=True)
            continue
        finally:
            for k, old in saved.items():
                if old is None:
                    os.environ.pop(k, None)
                else:
                    os.environ[k] = old
        sb = ex.scratch_bytes()
        scr = torch.empty(sb, dtype=torch.uint8, device="cuda") if sb else None
        ex.run(dev, scr, 3)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        ex.run(dev, scr, steps)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / steps
        ex.set_profiling(True)
        ex.run(dev, scr, steps)
        torch.cuda.synchronize()
        gms, _ = ex.group_times()
        gi = [ex.group_info(g) for g in range(ex.info().n_groups)]
        jit = [prog.jit_check(plan, g, kf.Target(**kw))[0] for g in range(len(gi))] if os.environ.get("AB_JIT") else None
        print(json.dumps({"variant": v, "ms_per_step": round(ms, 4), "jit_regs": jit,
                          "groups": [(g.name.decode(), round(t / steps, 4), g.regs, g.smem_bytes) for g, t in zip(gi, gms)]}),
              flush=True)
        del ex, scr


if __name__ == "__main__":
    main()
