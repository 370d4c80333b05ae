"""Sampled-window parity at full size (test infrastructure, like the rest of oracle/).

An output window of a program after `nsteps` steps depends on its inputs only through a
dependency cone of xy radius R = sum over the steps of the longest chain of kernel footprints
(each kernel's largest |di|, |dj| added along its reads).  Cropping the window plus a margin
M > R out of the global inputs -- wrapped on periodic axes, the crop's own boundary FROZEN with
the true neighbours as its ghost cells -- gives a small program whose interior window the
oracle computes exactly as the global run would (no arithmetic of the method here: index
bookkeeping for interp.run).  Used by tests/test_gpu_fullsize.py and bench.py's parity leg."""
from __future__ import annotations

from typing import Dict, Tuple

import numpy as np

from workloads.program import BC_FROZEN, Program


def dependency_radius(desc: Program, nsteps: int) -> int:
    """xy radius of the cone through which an output after `nsteps` depends on the inputs."""
    rad = {x: 0 for x in range(len(desc.arrays))}
    for _ in range(nsteps):
        for kern in desc.kernels:
            r = max(rad[a] + max(max(abs(d[0]), abs(d[1])) for d in offs) for a, offs in kern.reads().items())
            for o in kern.writes():
                rad[o] = max(rad[o], r)
    return max(rad.values())


def crop(desc: Program, arrays: Dict[str, np.ndarray], x0: int, y0: int, w: int, margin: int
         ) -> Tuple[Program, Dict[str, np.ndarray]]:
    """Window [x0, x0+w) x [y0, y0+w) plus margin, wrapped on the xy axes, as a frozen-xy
    sub-problem (its ghost cells are the true neighbours)."""
    nx, ny, nz = desc.n
    g = desc.ghost
    W = w + 2 * margin
    xi = (np.arange(-margin - g[0], w + margin + g[0]) + x0) % nx + g[0]
    yi = (np.arange(-margin - g[1], w + margin + g[1]) + y0) % ny + g[1]
    sub = desc.with_(n=(W, W, nz), bc=(BC_FROZEN, BC_FROZEN, desc.bc[2]))
    return sub, {nm: np.ascontiguousarray(a[:, yi][:, :, xi]) for nm, a in arrays.items()}


def window(desc: Program, arr: np.ndarray, x0: int, y0: int, w: int) -> np.ndarray:
    """Interior planes of the global window [x0, x0+w) x [y0, y0+w) (wrapped)."""
    nx, ny, nz = desc.n
    g = desc.ghost
    xs = (np.arange(x0, x0 + w) % nx) + g[0]
    ys = (np.arange(y0, y0 + w) % ny) + g[1]
    return arr[g[2]:g[2] + nz][:, ys][:, :, xs]


def crop_window(sub: Program, arr: np.ndarray, w: int, margin: int) -> np.ndarray:
    """The window inside a crop made by `crop`."""
    g = sub.ghost
    nz = sub.n[2]
    return arr[g[2]:g[2] + nz, g[1] + margin:g[1] + margin + w, g[0] + margin:g[0] + margin + w]
