"""ncu driver: run `steps` steps of one weather plan (labels JSON, or hgga/hand) with one target.

  ncu ... python tools/prof_plan.py '<plan>' '<target json>' [steps] ['<per-group configs json>']

The optional per-group configs are bench.py's config.per_group_launch_config
([tile, stages, zunroll, ringunroll, minblocks, canvas_ld] per group).
"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_wahibm14_b200 as kf
from workloads import programs as P, data as D
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ab import HGGA

desc = P.weather(n=(512, 512, 128))
prog = kf.Program(desc)
which = sys.argv[1]
plan = {"hgga": HGGA, "hand": P.weather_hand_plan(desc)}.get(which) or json.loads(which)
kw = {k: (tuple(v) if isinstance(v, list) else v) for k, v in json.loads(sys.argv[2] if len(sys.argv) > 2 else "{}").items()}
steps = int(sys.argv[3]) if len(sys.argv) > 3 else 2
gt = None
if len(sys.argv) > 4:
    gt = [kf.Target(**dict(kw, tile=tuple(c[0]), stages=c[1], zunroll=c[2], ringunroll=c[3], minblocks=c[4],
                           canvas_ld=c[5] if len(c) > 5 else 1, pblock=(c[6] if len(c) > 6 else 1, 1),
                           pair_zq=c[7] if len(c) > 7 else 1))
          for c in json.loads(sys.argv[4])]
ex = kf.Exec(prog, plan, kf.Target(**kw), group_targets=gt)
ex.set_graph(False)
dev = kf.device_arrays(prog, D.weather_inputs(desc, 3))
sb = ex.scratch_bytes()
scr = torch.empty(sb, dtype=torch.uint8, device="cuda") if sb else None
ex.run(dev, scr, steps)
torch.cuda.synchronize()
print("done", [(ex.group_info(g).name.decode(), ex.group_info(g).threads, ex.group_info(g).regs, ex.group_info(g).smem_bytes)
               for g in range(ex.info().n_groups)])
