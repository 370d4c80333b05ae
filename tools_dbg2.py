import os, sys, numpy as np
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import torch
import paper_conf_sc_wahibm14_b200 as kf
from oracle import interp, enum as En, graph as G
from workloads import programs as P, data as D
from workloads.program import *
from tests.gpu_util import run_kf, compare, bits
def show(desc, got, ref):
    for nm in [nm for x,(nm,_) in enumerate(desc.arrays) if not G.writers(desc,x) or G.step_live(desc,x)]:
        g, o = got[nm], ref[nm]
        bad = np.argwhere(bits(g) != bits(o))
        if len(bad):
            gz,gy,gx = desc.ghost
            print("   ", nm, "nbad", len(bad), "first(z,y,x interior coords)", [tuple(int(v) for v in (b - np.array([gz,gy,gx]))) for b in bad[:4]], "got", g[tuple(bad[0])], "ref", o[tuple(bad[0])])
cases = []
for seed in range(6):
    rng = np.random.default_rng(1000 + seed)
    bc = tuple(int(x) for x in rng.integers(0, 2, size=3))
    flags = [0, PROG_RELAX_EXPANDABLE, PROG_RELAX_ALL][seed % 3]
    dtype = DT_F32 if seed % 2 else DT_F64
    n = tuple(int(x) for x in rng.integers(9, 40, size=3))
    desc = P.random_program(2000 + seed, nk=5, na=4, n=n, dtype=dtype, bc=bc, flags=flags, max_r=1 + seed % 2)
    inputs = D.uniform(desc, seed)
    for nsteps in (1, 2):
        ref = interp.run(desc, inputs, nsteps)
        got, ex = run_kf(desc, list(range(5)), inputs, nsteps, kf.Target(tile=(16,16,0)))
        print("seed", seed, "bc", bc, "flags", flags, "n", n, "steps", nsteps, "ok" if not compare(desc, got, ref) else "BAD")
        show(desc, got, ref)
# simple periodic test: shift kernel
b = Builder("shift", DT_F64, (20, 12, 8), (1, 1, 1), (BC_PERIODIC,) * 3)
a = b.array("a"); t = b.array("t")
b.kernel("s", (t, a[-1, 0, 0])); b.kernel("c", (a, t.c))
desc = b.build(); inputs = D.uniform(desc, 3)
for plan in ([0,1],):
    ref = interp.run(desc, inputs, 1); got, ex = run_kf(desc, plan, inputs, 1)
    print("shift", plan, compare(desc, got, ref)); show(desc, got, ref)
