"""Sweep tile/stages/threads for a plan of the weather workload in one process (inputs generated once)."""
import itertools, json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_wahibm14_b200 as kf
from workloads import programs as P, data as D

def main():
    plan_kind = sys.argv[1] if len(sys.argv) > 1 else "hand"
    configs = json.loads(sys.argv[2]) if len(sys.argv) > 2 else [[[32, 16, 0], 2, 256]]
    from workloads.program import PROG_RELAX_ALL, PROG_RELAX_EXPANDABLE
    desc = P.weather(n=(512, 512, 128), relax=PROG_RELAX_ALL if plan_kind.endswith("_all") else PROG_RELAX_EXPANDABLE)
    prog = kf.Program(desc)
    inputs = D.weather_inputs(desc, 3)
    dev = kf.device_arrays(prog, inputs)
    del inputs
    out = []
    for cfg in configs:
        tile, stages, threads = cfg[:3]
        zu = cfg[3] if len(cfg) > 3 else 1
        pb = cfg[4] if len(cfg) > 4 else [1, 1]
        ru = cfg[5] if len(cfg) > 5 else 0
        gw = cfg[6] if len(cfg) > 6 else 0
        if len(cfg) > 7:   # codegen A/B knob: max z-queue registers per thread
            os.environ["KF_ZQ_MAX"] = str(cfg[7])
        tgt = kf.Target(tile=tile, stages=stages, threads=threads, zunroll=zu, pblock=pb, ringunroll=ru, ghostwrite=gw)
        if plan_kind == "hand":
            plan = P.weather_hand_plan(desc)
        elif plan_kind == "unfused":
            plan = list(range(44))
        elif plan_kind.startswith("hgga"):
            plan, _ = prog.search(kf.SEARCH_HGGA, tgt, seed=1)
        elif plan_kind.startswith("time"):
            plan, _ = prog.search(kf.SEARCH_GREEDY_TIME, tgt)
        else:
            plan, _ = prog.search(kf.SEARCH_GREEDY, tgt)
        try:
            ex = kf.Exec(prog, plan, tgt)
        except Exception as e:
            print(json.dumps({"tile": tile, "stages": stages, "threads": threads, "error": str(e)[:200]}), flush=True)
            continue
        sb = ex.scratch_bytes()
        scr = torch.empty(sb, dtype=torch.uint8, device="cuda") if sb else None
        ex.run(dev, scr, 3)
        torch.cuda.synchronize()
        ex.set_profiling(True)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        ex.run(dev, scr, 10)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 10
        gms, _ = ex.group_times()
        info = ex.info()
        per, _, _ = prog.project(plan, tgt)
        r = {"plan": plan_kind, "model_ms": sum(g.t_model_s for g in per) * 1e3, "tile": tile, "stages": stages, "threads": threads, "zunroll": zu, "pblock": pb, "ringunroll": ru, "ghostwrite": gw, "zq_max": os.environ.get("KF_ZQ_MAX"), "ms_per_step": ms,
             "TBps": info.compulsory_bytes_per_step / ms / 1e9,
             "groups": [(ex.group_info(g).name.decode(), round(gms[g] / 10, 4),
                         round(ex.group_info(g).bytes_per_launch / (gms[g] / 10) / 1e9, 2),
                         ex.group_info(g).smem_bytes, ex.group_info(g).regs) for g in range(len(gms))]}
        print(json.dumps(r), flush=True)
        del ex, scr

main()
