"""Helpers for the GPU parity tests: run a plan through the C ABI and compare with the oracle."""
import numpy as np

from oracle import graph as G


def kept_arrays(desc):
    """Arrays whose contents are specified after a run: read-only, never written, or step-live
    (TEMP arrays are unspecified under fused plans, R15)."""
    return [nm for x, (nm, _) in enumerate(desc.arrays) if not G.writers(desc, x) or G.step_live(desc, x)]


def run_kf(desc, plan, inputs, nsteps, target=None, graph=True, params=None):
    import torch

    import paper_conf_sc_wahibm14_b200 as kf
    prog = kf.Program(desc)
    ex = kf.Exec(prog, plan, target)
    ex.set_graph(graph)
    dev = kf.device_arrays(prog, inputs)
    sb = ex.scratch_bytes()
    scratch = torch.empty(sb, dtype=torch.uint8, device="cuda") if sb else None
    ex.run(dev, scratch, nsteps, params)
    torch.cuda.synchronize()
    return kf.host_arrays(prog, dev), ex


def bits(a):
    return a.view(np.uint32 if a.dtype == np.float32 else np.uint64)


def defined_cells(desc):
    """Cells whose value is specified after a run: the interior, plus ghost cells of FROZEN axes
    (never written).  Ghost layers of PERIODIC axes are overwritten by the library's wrap fill
    (kf.h, R9) while the oracle wraps on reads, so they are not compared."""
    nx, ny, nz = desc.n
    gx, gy, gz = desc.ghost
    m = np.ones(desc.padded_shape(), dtype=bool)
    for a, (n, g) in enumerate(((nx, gx), (ny, gy), (nz, gz))):
        if desc.bc[a] == 1 and g > 0:
            sl = [slice(None)] * 3
            sl[2 - a] = slice(0, g)
            m[tuple(sl)] = False
            sl[2 - a] = slice(g + n, None)
            m[tuple(sl)] = False
    return m


def compare(desc, got, ref, names=None, rtol32=2e-6):
    """fp64: bit-exact.  fp32: normwise max|g-o| <= 2e-6 * max|o| per array (north_star), and we
    also require bit-exactness because both sides perform identical IEEE operations."""
    bad = []
    mask = defined_cells(desc)
    for nm in (names or kept_arrays(desc)):
        g, o = got[nm][mask], ref[nm][mask]
        if g.dtype == np.float32:
            scale = float(np.max(np.abs(o))) if o.size else 0.0
            err = float(np.max(np.abs(g.astype(np.float64) - o.astype(np.float64)))) if o.size else 0.0
            if not err <= rtol32 * max(scale, 1e-30):
                bad.append((nm, "tol", err, scale))
                continue
        if not np.array_equal(bits(g), bits(o)):
            d = np.argwhere(bits(g) != bits(o))
            bad.append((nm, "bits", int(len(d)), tuple(int(v) for v in d[0])))
    return bad
