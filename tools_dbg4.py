import os, sys, numpy as np
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import torch
import paper_conf_sc_wahibm14_b200 as kf
from oracle import interp, enum as En, graph as G
from workloads import programs as P, data as D
from workloads.program import *
from tests.gpu_util import compare, run_kf, bits, defined_cells
from tests.test_dist import _run_loopback
seed = 3
desc = P.random_program(300 + seed, nk=4, na=4, n=(24, 18, 7), dtype=DT_F32, bc=(BC_PERIODIC, BC_PERIODIC, BC_FROZEN), flags=PROG_RELAX_ALL, max_r=2)
print([(k.name, k.writes(), k.reads()) for k in desc.kernels])
inputs = D.uniform(desc, seed)
ref = interp.run(desc, inputs, 2)
plan = [0,0,0,0]
got, _ = run_kf(desc, plan, inputs, 2, kf.Target(tile=(8,4,0)))
print("single", compare(desc, got, ref))
for px, py in ((1,1),(2,1),(1,3),(2,3)):
    got = _run_loopback(desc, plan, inputs, 2, px, py, kf.Target(tile=(8,4,0)))
    b = compare(desc, got, ref)
    print(px, py, b)
    m = defined_cells(desc)
    for nm in set(x[0] for x in b):
        diff = (bits(got[nm]) != bits(ref[nm])) & m
        idx = np.argwhere(diff); g = desc.ghost
        print("  ", nm, len(idx), "z", idx[:,0].min()-g[2], idx[:,0].max()-g[2], "y", sorted(set((idx[:,1]-g[1]).tolist()))[:20], "x", sorted(set((idx[:,2]-g[0]).tolist()))[:30])
for nsteps in (1,):
    ref1 = interp.run(desc, inputs, 1)
    got = _run_loopback(desc, plan, inputs, 1, 2, 1, kf.Target(tile=(8,4,0)))
    print("1 step 2x1", compare(desc, got, ref1))
