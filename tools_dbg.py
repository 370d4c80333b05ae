import os, sys, numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import paper_conf_sc_wahibm14_b200 as kf
from workloads import programs as P, data as D
desc = P.tiny(n=(32,16,8))
prog = kf.Program(desc)
plan = [int(x) for x in sys.argv[1].split(",")] if len(sys.argv) > 1 else [0,1,2]
ex = kf.Exec(prog, plan)
ex.set_graph(False)
dev = kf.device_arrays(prog, D.uniform(desc, 1))
print("launching", plan, [ex.group_info(g).name for g in range(ex.info().n_groups)], flush=True)
ex.run(dev, None, 1)
torch.cuda.synchronize()
print("ok", flush=True)
