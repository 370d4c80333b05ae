"""Small driver for ncu: runs `steps` steps of a weather plan (default: hand plan) at full size."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_wahibm14_b200 as kf
from workloads import programs as P, data as D
plan_kind = sys.argv[1] if len(sys.argv) > 1 else "hand"
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 2
tile = tuple(int(v) for v in (sys.argv[3] if len(sys.argv) > 3 else "32,16,0").split(","))
desc = P.weather(n=(512, 512, 128))
prog = kf.Program(desc)
tgt = kf.Target(tile=tile)
plan = {"hand": lambda: P.weather_hand_plan(desc), "unfused": lambda: list(range(44)),
        "best": lambda: prog.search(kf.SEARCH_GREEDY, tgt)[0]}[plan_kind]()
ex = kf.Exec(prog, plan, tgt)
ex.set_graph(False)
dev = kf.device_arrays(prog, D.weather_inputs(desc, 3))
sb = ex.scratch_bytes()
scr = torch.empty(sb, dtype=torch.uint8, device="cuda") if sb else None
ex.run(dev, scr, steps)
torch.cuda.synchronize()
print("done", [ex.group_info(g).name.decode() for g in range(ex.info().n_groups)])
