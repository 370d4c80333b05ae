import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_wahibm14_b200 as kf, sys
from workloads import programs
prog = kf.Program(programs.weather(n=(512,512,128)))
plan=[0, 0, 0, 1, 1, 1, 1, 1, 1, 2, 2, 2, 2, 2, 2, 0, 2, 0, 0, 0, 0, 1, 1, 1, 1, 2, 2, 3, 2, 2, 4, 4, 3, 5, 5, 4, 4, 3, 5, 5, 4, 4, 3, 5]
t = kf.Target(tile=(32,8,64))
r = prog.jit_check(plan, 0, t); print("jit", r[0], r[1])
ex = kf.Exec(prog, plan, t)
print("exec before run", [(ex.group_info(g).regs, ex.group_info(g).local_bytes) for g in range(6)])
import torch
from workloads import data as D
dev = kf.device_arrays(prog, D.weather_inputs(prog.desc, 3))
sb = ex.scratch_bytes(); scr = torch.empty(sb, dtype=torch.uint8, device="cuda") if sb else None
ex.run(dev, scr, 1); torch.cuda.synchronize()
print("exec after run", [(ex.group_info(g).regs, ex.group_info(g).local_bytes) for g in range(6)])
