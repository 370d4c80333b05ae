"""Seeded synthetic inputs (no arithmetic of the method lives here).

Arrays are numpy arrays in the *logical ghosted* shape (nz+2gz, ny+2gy, nx+2gx),
x fastest, in the program dtype.  Ghost cells are filled too: on frozen axes
they are the user-initialised boundary values the method never writes.
The same arrays are handed to the oracle and uploaded to the GPU.
"""
from __future__ import annotations

from typing import Dict

import numpy as np

from .program import DT_F32, Program


def np_dtype(prog: Program):
    return np.float32 if prog.dtype == DT_F32 else np.float64


def uniform(prog: Program, seed: int, lo=-1.0, hi=1.0) -> Dict[str, np.ndarray]:
    rng = np.random.default_rng(seed)
    shp = prog.padded_shape()
    return {nm: rng.uniform(lo, hi, size=shp).astype(np_dtype(prog)) for nm, _ in prog.arrays}


def coords(prog: Program, centred=True):
    """Integer interior coordinates (i, j, k) over the ghosted shape (ghosts get -g..-1, n..n+g-1)."""
    nx, ny, nz = prog.n
    gx, gy, gz = prog.ghost
    k, j, i = np.meshgrid(np.arange(-gz, nz + gz), np.arange(-gy, ny + gy), np.arange(-gx, nx + gx),
                          indexing="ij")
    if centred:
        i, j, k = i - nx // 2, j - ny // 2, k - nz // 2
    return i, j, k


def quadratic(prog: Program, seed: int = 0) -> Dict[str, np.ndarray]:
    """Closed-form variant of config 1: u = i^2 + 2 j^2 + 3 k^2 everywhere (incl. ghosts),
    v ghosts = 12 (= L7 of u), other arrays 0.  Exact in fp32 on 32^3 (|u| < 2^24)."""
    i, j, k = coords(prog)
    dt = np_dtype(prog)
    out = {}
    for nm, _ in prog.arrays:
        out[nm] = np.zeros(prog.padded_shape(), dtype=dt)
    out["u"] = (i * i + 2 * j * j + 3 * k * k).astype(dt)
    out["v"] = np.full(prog.padded_shape(), 12.0, dtype=dt)
    return out


def fig3_inputs(prog: Program, seed: int) -> Dict[str, np.ndarray]:
    """Fig. 3 program inputs; Q and V in [1, 2] because kernels D and E divide by them."""
    out = uniform(prog, seed)
    rng = np.random.default_rng(seed + 1000)
    for nm in ("Q", "V"):
        out[nm] = rng.uniform(1.0, 2.0, size=prog.padded_shape()).astype(np_dtype(prog))
    return out


def weather_inputs(prog: Program, seed: int) -> Dict[str, np.ndarray]:
    """Smooth fields + 1e-3 noise: DENS in [0.9, 1.1], MOM in [-0.1, 0.1], RHOT ~ 300 DENS."""
    rng = np.random.default_rng(seed)
    shp = prog.padded_shape()
    dt = np_dtype(prog)
    nz, ny, nx = shp
    z, y, x = np.meshgrid(np.linspace(0, 2 * np.pi, nz, endpoint=False),
                          np.linspace(0, 2 * np.pi, ny, endpoint=False),
                          np.linspace(0, 2 * np.pi, nx, endpoint=False), indexing="ij")

    def smooth(amp, phase):
        return amp * np.sin(x + phase) * np.cos(y - phase) * np.cos(0.5 * z + phase)

    def noise(s=1e-3):
        return s * rng.standard_normal(shp)

    out = {nm: np.zeros(shp, dtype=dt) for nm, _ in prog.arrays}
    dens = 1.0 + smooth(0.08, 0.1) + noise()
    out["DENS"] = dens.astype(dt)
    out["DENS0"] = dens.astype(dt)
    for s, ph in (("MOMX", 0.3), ("MOMY", 0.7), ("MOMZ", 1.1)):
        m = smooth(0.08, ph) + noise()
        out[s] = m.astype(dt)
        out[s + "0"] = m.astype(dt)
    rhot = 300.0 * dens + noise(1e-2)
    out["RHOT"] = rhot.astype(dt)
    out["RHOT0"] = rhot.astype(dt)
    out["DENS_REF"] = (1.0 + 0.01 * np.cos(0.5 * z)).astype(dt)
    out["PRES_REF"] = (100.0 + np.cos(0.5 * z)).astype(dt)
    out["CORI"] = np.full(shp, 1.0e-4, dtype=dt)
    # TEMP arrays keep deterministic (zero-mean noise) ghosts so frozen-z reads are defined
    for nm, _ in prog.arrays:
        if not out[nm].any():
            out[nm] = noise(1e-3).astype(dt)
    return out


def inputs_for(prog: Program, seed: int) -> Dict[str, np.ndarray]:
    if prog.name == "fig3":
        return fig3_inputs(prog, seed)
    if prog.name == "weather":
        return weather_inputs(prog, seed)
    return uniform(prog, seed)
