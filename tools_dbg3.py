import os, sys, numpy as np
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import paper_conf_sc_wahibm14_b200 as kf
from oracle import interp, enum as En, graph as G, legality as L
from workloads import programs as P, data as D
from workloads.program import *
from tests.gpu_util import run_kf, compare, bits, defined_cells

def bad_of(desc, plan, inputs, nsteps, tile=(32,16,0), ref=None):
    ref = ref if ref is not None else interp.run(desc, inputs, nsteps)
    got, ex = run_kf(desc, plan, inputs, nsteps, kf.Target(tile=tile))
    return compare(desc, got, ref), got, ref

def isolate(desc, plan, inputs, nsteps, tile):
    ref = interp.run(desc, inputs, nsteps)
    gs = L.groups_of(plan)
    for gi, g in enumerate(gs):
        if len(g) < 2: continue
        p2 = list(range(len(desc.kernels)))
        for k in g: p2[k] = g[0]
        if L.validate(desc, p2)[0] != 0:
            print("group", gi, "alone is illegal", L.validate(desc, p2)); continue
        b, got, _ = bad_of(desc, p2, inputs, nsteps, tile, ref)
        print("group", gi, [desc.kernels[k].name for k in g], "->", b[:3])
        if b:
            # shrink: try removing kernels one at a time while still failing
            cur = list(g)
            changed = True
            while changed:
                changed = False
                for k in list(cur):
                    trial = [x for x in cur if x != k]
                    if len(trial) < 2: continue
                    p3 = list(range(len(desc.kernels)))
                    for x in trial: p3[x] = trial[0]
                    if L.validate(desc, p3)[0] != 0: continue
                    b3, _, _ = bad_of(desc, p3, inputs, nsteps, tile, ref)
                    if b3:
                        cur = trial; changed = True; break
            print("  minimal failing group:", [(k, desc.kernels[k].name) for k in cur])
            p3 = list(range(len(desc.kernels)))
            for x in cur: p3[x] = cur[0]
            b3, got, ref2 = bad_of(desc, p3, inputs, nsteps, tile, ref)
            print("  ", b3)
            m = defined_cells(desc)
            for nm in set(x[0] for x in b3):
                diff = (bits(got[nm]) != bits(ref2[nm])) & m
                idx = np.argwhere(diff)
                gz,gy,gx = desc.ghost
                print("   ", nm, len(idx), "z range", idx[:,0].min()-gz, idx[:,0].max()-gz, "y", idx[:,1].min()-gy, idx[:,1].max()-gy, "x", idx[:,2].min()-gx, idx[:,2].max()-gx)
            ex = kf.Exec(kf.Program(desc), p3, kf.Target(tile=tile))
            open("gpurun_out/min_group.cu", "w").write(ex.group_source(L.canonical(p3)[cur[0]]))
            return

seed = 10
rng = np.random.default_rng(1000 + seed)
bc = tuple(int(x) for x in rng.integers(0, 2, size=3))
flags = [0, PROG_RELAX_EXPANDABLE, PROG_RELAX_ALL][seed % 3]
dtype = DT_F32 if seed % 2 else DT_F64
n = tuple(int(x) for x in rng.integers(9, 40, size=3))
desc = P.random_program(2000 + seed, nk=5, na=4, n=n, dtype=dtype, bc=bc, flags=flags, max_r=1 + seed % 2)
print("seed10", bc, flags, n, [ (k.name, k.writes(), k.reads()) for k in desc.kernels])
inputs = D.uniform(desc, seed)
nsteps = 1 + seed % 3
isolate(desc, [0,0,1,0,1], inputs, nsteps, (8,4,6))
desc = P.weather(n=(48, 40, 12))
inputs = D.inputs_for(desc, 3)
plan_g, _ = kf.Program(desc).search(kf.SEARCH_GREEDY)
isolate(desc, plan_g, inputs, 1, (32,16,0))
