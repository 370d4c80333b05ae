#!/usr/bin/env python
"""Benchmark of the fused stencil-program hot path on B200 (BASELINE.json metric).

One *step* = one pass of the whole hot path over the program: every fused group of the
plan in quotient-topological order (periodic ghosts written by the producing groups; halo
exchanges between ranks at N > 1) = one timestep of the 44-kernel / 31-array weather-shaped
program (BASELINE config 3, 512x512x128 fp64 per GPU).

Printed JSON (rank 0, one line): metric/value = grid-points*steps/s of the fused plan with
inputs resident in HBM (CUDA events on the launch stream, max over ranks), plus the roofline of
the dominant group kernel, per-group measured vs projected times (NEXT-2), the parity of the
timed configuration on sampled windows against the oracle, the oracle's CPU baseline (1 core and
all cores), the end-to-end number through kf_run_host (host buffers, copies inside the timed
region), the unfused plan's speed (speedup vs unfused), Fusion Efficiency (Eq. 12) and SM clocks.

  python bench.py [--gpus N --steps K --warmup W] [--workload weather|weak|stress|suite|tiny]
  python bench.py --workload suite --all-plans        # config 2: every legal plan timed
  python bench.py --impl reference ...                # the oracle on host cores, same metric/config

--gpus N > 1 without a launcher re-executes itself under torch.distributed.run (one rank per
GPU); with a launcher WORLD_SIZE must equal N.  Workloads: weather = config 3 (weak scaling,
512x512x128 per GPU), weak = config 4 (1024x1024x128 per GPU), stress = config 5 (768^3 global,
strong scaling over a px x py split), suite = config 2 (256^3 fp32), tiny = config 1.
"""
from __future__ import annotations

import argparse
import json
import os
import socket
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

METRIC = "fused-program grid-pts·steps/s"
UNIT = "grid-pts·steps/s"


def grid_for(world):
    return {1: (1, 1), 2: (2, 1), 4: (2, 2), 8: (4, 2)}.get(world, (world, 1))


# ---------------------------------------------------------------- workloads
class Workload:
    """The per-rank (local) program, its input generator and labels.  `global_n` is the grid the
    whole job covers (weak: per-GPU grid x ranks; strong: fixed)."""

    def __init__(self, name: str, world: int):
        from workloads import programs
        self.name = name
        px, py = grid_for(world)
        self.scaling = "weak"
        self.tile_grid = None
        if name == "weather":
            self.desc = programs.weather(n=(512, 512, 128))
            self.gen = "weather"
            self.tkw = dict(tile=(32, 8, 64))
            self.label = "weather-44k31a-512x512x128-fp64 per GPU (BASELINE config 3)"
        elif name == "weak":
            # config 4: 1024x1024x128 per GPU; fields generated at 512x512x128 and tiled 2x2 on the device
            self.desc = programs.weather(n=(1024, 1024, 128))
            self.gen = "weather_tiled"
            self.tile_grid = (512, 512, 128)
            self.tkw = dict(tile=(32, 8, 64))
            self.label = "weather-44k31a-1024x1024x128-fp64 per GPU (BASELINE config 4, weak)"
        elif name == "weather_small":
            self.desc = programs.weather(n=(128, 128, 64))
            self.gen = "weather"
            self.tkw = dict(tile=(32, 16, 0))
            self.label = "weather-44k31a-128x128x64-fp64"
        elif name == "suite":
            self.desc = programs.gen_suite(seed=0)
            self.gen = "uniform"
            self.tkw = dict(tile=(32, 8, 0))
            self.label = "suite-10k8a-256^3-fp32 (BASELINE config 2, gen_suite seed 0)"
        elif name == "tiny":
            self.desc = programs.tiny()
            self.gen = "uniform"
            self.tkw = dict(tile=(32, 16, 0))
            self.label = "tiny-3k3a-32^3-fp32 (BASELINE config 1)"
        elif name == "fig3":
            self.desc = programs.fig3(n=(512, 512, 128))
            self.gen = "fig3"
            self.tkw = dict(tile=(32, 16, 0))
            self.label = "fig3-6k-512x512x128-fp64"
        elif name == "stress":
            # config 5: 768^3 global, strong scaling over the px x py process grid
            if 768 % px or 768 % py:
                raise SystemExit(f"stress: 768 not divisible by the process grid {px}x{py}")
            self.desc = programs.stress(m=2, n=(768 // px, 768 // py, 768))
            self.gen = "device_uniform"
            self.tkw = dict(tile=(32, 8, 0), max_halo=16)
            self.scaling = "strong"
            self.label = f"stress-2fields-L25xL25-768^3-fp64 (config 5, strong; local {768 // px}x{768 // py}x768)"
        else:
            raise SystemExit(f"unknown workload {name}")
        self.world = world
        # weak: every rank owns a full per-GPU grid; strong: the local grids partition the global one
        self.global_npts = self.desc.npts * world

    def inputs(self, prog, rank, device_ok=True):
        """Device tensors (kf layout) of the rank's seeded synthetic inputs."""
        import torch
        import paper_conf_sc_wahibm14_b200 as kf
        from workloads import data, programs
        seed = 3 + rank
        if self.gen == "device_uniform":
            L = prog.layout()
            gdev = torch.Generator(device="cuda").manual_seed(seed)
            dt = torch.float64 if self.desc.dtype == 1 else torch.float32
            return [torch.rand(L.elems, generator=gdev, device="cuda", dtype=dt) * 2 - 1 for _ in self.desc.arrays], None
        if self.gen == "weather_tiled":
            small = programs.weather(n=self.tile_grid)
            sin = data.weather_inputs(small, seed)
            return tile_to_device(prog, small, sin), None
        if self.gen == "weather":
            inp = data.weather_inputs(self.desc, seed)
        elif self.gen == "fig3":
            inp = data.fig3_inputs(self.desc, seed)
        else:
            inp = data.uniform(self.desc, seed)
        return kf.device_arrays(prog, inp), inp


def tile_to_device(prog, small, sin):
    """Periodic xy tiling of a small field set into the program's (larger) grid, on the device:
    interior (k, j, i) <- small interior (k, j mod ny_s, i mod nx_s); x/y ghosts wrap; z ghosts are
    the small grid's (plumbing: synthetic inputs only)."""
    import torch
    d = prog.desc
    L = prog.layout()
    g = d.ghost
    nxs, nys, nzs = small.n
    assert nzs == d.n[2] and small.ghost == d.ghost
    xi = torch.tensor([(i % nxs) + g[0] for i in range(-g[0], d.n[0] + g[0])], device="cuda")
    yi = torch.tensor([(j % nys) + g[1] for j in range(-g[1], d.n[1] + g[1])], device="cuda")
    out = []
    for nm, _ in d.arrays:
        s = torch.from_numpy(sin[nm]).to("cuda")
        big = s[:, yi][:, :, xi]
        flat = torch.zeros(L.elems, dtype=s.dtype, device="cuda")
        v = flat.view(d.n[2] + 2 * g[2], L.rows, L.pitch)
        v[:, :, L.xoff - g[0]:L.xoff + d.n[0] + g[0]] = big
        out.append(flat)
        del s, big
    return out


def plan_candidates(prog, target):
    """Candidate plans for measured selection: the paper's search (HGGA) on the projected
    time with five seeds (two, plus brute force, for small programs) and on compulsory bytes, greedy
    merging on projected time, and (weather) the App. A.4 hand plan.  Deduplicated by canonical
    labelling."""
    import paper_conf_sc_wahibm14_b200 as kf
    out, seen = [], set()

    def add(plan, kind):
        canon, m = [], {}
        for g in plan:
            canon.append(m.setdefault(g, len(m)))
        if tuple(canon) not in seen:
            seen.add(tuple(canon))
            out.append((canon, kind))
    if prog.nk <= 10:
        add(prog.search(kf.SEARCH_BRUTE_TIME, target)[0], "brute-force on projected time")
        add(prog.search(kf.SEARCH_BRUTE, target)[0], "brute-force on compulsory bytes")
        add(prog.search(kf.SEARCH_GREEDY_TIME, target)[0], "greedy merging on projected time")
        for seed in (1, 2):
            add(prog.search(kf.SEARCH_HGGA, target, seed=seed)[0], f"HGGA (seed {seed}) on the resource-aware projected time")
    else:
        for seed in (1, 2, 3, 4, 5):
            add(prog.search(kf.SEARCH_HGGA, target, seed=seed)[0], f"HGGA (seed {seed}) on the resource-aware projected time")
        add(prog.search(kf.SEARCH_HGGA_BYTES, target, seed=1)[0], "HGGA (seed 1) on compulsory bytes")
        add(prog.search(kf.SEARCH_GREEDY_TIME, target)[0], "greedy merging on projected time")
    if prog.desc.name == "weather":
        from workloads.programs import weather_hand_plan
        add(weather_hand_plan(prog.desc), "hand plan (App. A.4)")
    return out


def time_exec(ex, dev, steps, warm=2):
    import torch
    sb = ex.scratch_bytes()
    scr = torch.empty(sb, dtype=torch.uint8, device="cuda") if sb else None
    ex.run(dev, scr, warm)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    ex.run(dev, scr, steps)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / steps


def select_plan(prog, target, dev, steps=5):
    """Measured selection among plan_candidates(): every candidate is compiled with the default
    launch configuration and timed (CUDA events, `steps` steps after 2 warm-up steps); the
    fastest is kept.  The projection ranks plans inside the search; the measurement decides
    between the few it proposes."""
    import torch
    import paper_conf_sc_wahibm14_b200 as kf
    res = []
    for plan, kind in plan_candidates(prog, target):
        try:
            ex = kf.Exec(prog, plan, target)
        except Exception as e:   # an illegal candidate for this target: skip it
            res.append((float("inf"), plan, kind + f" (failed: {str(e)[:80]})", []))
            continue
        ms = time_exec(ex, dev, steps)
        # per-group times of the candidate under the default launch configuration (NEXT-2 data:
        # measured vs projected for every group the searches propose)
        sb = ex.scratch_bytes()
        scr = torch.empty(sb, dtype=torch.uint8, device="cuda") if sb else None
        ex.set_profiling(True)
        ex.run(dev, scr, steps)
        torch.cuda.synchronize()
        gms, _ = ex.group_times()
        ex.set_profiling(False)
        per, _, _ = prog.project(plan, target)
        groups = [{"kernels": [k for k in range(len(plan)) if plan[k] == g], "ms": gms[g] / steps, "t_model_ms": per[g].t_model_s * 1e3,
                   "t_bytes_ms": per[g].t_s * 1e3, "regs": ex.group_info(g).regs} for g in range(len(gms))]
        res.append((ms, plan, kind, groups))
        del ex, scr
    best = min(res, key=lambda r: r[0])
    ranked = [(plan, kind) for ms, plan, kind, _ in sorted(res, key=lambda r: r[0]) if ms < float("inf")]
    return best[1], best[2] + " (fastest of the measured candidates)", [
        {"plan": kind, "ms_per_step": round(ms, 4), "groups": len(set(plan)), "labels": plan, "per_group": g}
        for ms, plan, kind, g in res], ranked


def choose_plan(prog, target, which: str):
    import paper_conf_sc_wahibm14_b200 as kf
    n = prog.nk
    if which == "unfused":
        return list(range(n)), "unfused (singletons)"
    if which == "hand":
        from workloads.programs import weather_hand_plan
        return weather_hand_plan(prog.desc), "hand plan (App. A.4)"
    if which.startswith("["):   # explicit labels, e.g. config.plan_labels of an earlier run
        return [int(v) for v in json.loads(which)], "given labels"
    method = kf.SEARCH_BRUTE_TIME if n <= 10 else kf.SEARCH_HGGA
    plan, _ = prog.search(method, target, seed=1)
    return plan, ("brute-force on projected time" if method == kf.SEARCH_BRUTE_TIME
                  else "HGGA search (seed 1) on the resource-aware projected time")


# ---------------------------------------------------------------- clocks
class ClockSampler:
    """SM clock and clock-event reasons sampled through NVML every 5 ms DURING the timed region
    (a thread started before it, stopped after it); only samples taken while the region ran count."""
    REASONS = (("hw_slowdown", "nvmlClocksEventReasonHwSlowdown"),
               ("hw_thermal_slowdown", "nvmlClocksEventReasonHwThermalSlowdown"),
               ("sw_thermal_slowdown", "nvmlClocksEventReasonSwThermalSlowdown"),
               ("sw_power_cap", "nvmlClocksEventReasonSwPowerCap"),
               ("hw_power_brake", "nvmlClocksEventReasonHwPowerBrakeSlowdown"))

    def __init__(self, index: int):
        self.index = index
        self.samples = []
        self.err = None
        self.h = None
        self.stop = threading.Event()
        self.t0 = self.t1 = None

    def __enter__(self):
        try:
            import pynvml
            import torch
            self.nv = pynvml
            pynvml.nvmlInit()
            try:
                uuid = str(torch.cuda.get_device_properties(self.index).uuid)
                self.h = pynvml.nvmlDeviceGetHandleByUUID(uuid if uuid.startswith("GPU-") else "GPU-" + uuid)
            except Exception:
                self.h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.th = threading.Thread(target=self._loop, daemon=True)
            self.th.start()
        except Exception as e:  # no NVML: reported as unavailable, never guessed
            self.err = f"{type(e).__name__}: {e}"
            self.h = None
        return self

    def mark_start(self):
        # the sampler must be running before the timed region starts (short regions: tens of ms)
        t_wait = time.perf_counter()
        while self.h is not None and not self.samples and time.perf_counter() - t_wait < 1.0:
            time.sleep(0.001)
        self.t0 = time.perf_counter()

    def mark_end(self):
        self.t1 = time.perf_counter()

    def _loop(self):
        nv = self.nv
        while not self.stop.is_set():
            try:
                t = time.perf_counter()
                sm = nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM)
                rs = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                self.samples.append((t, sm, rs))
            except Exception as e:
                self.err = f"{type(e).__name__}: {e}"
                return
            time.sleep(0.002)

    def __exit__(self, *a):
        self.stop.set()
        if self.h is not None:
            self.th.join(timeout=2)

    def summary(self):
        if self.h is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"], "error": self.err}
        t0 = self.t0 if self.t0 is not None else float("-inf")
        t1 = self.t1 if self.t1 is not None else float("inf")
        win = [s for s in self.samples if t0 <= s[0] <= t1]
        if not win:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": ["no sample in the timed region"]}
        sm = sorted(s[1] for s in win)
        reasons = set()
        for _, _, rs in win:
            for nm, attr in self.REASONS:
                if rs & getattr(self.nv, attr, 0):
                    reasons.add(nm)
        return {"sm_mhz": sm[len(sm) // 2], "sm_max_mhz": self.max_mhz, "reasons": sorted(reasons),
                "samples": len(win), "source": "NVML, every 2 ms, inside the timed region"}


def measured_peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return None


def ncu_traffic(kernel_name: str):
    """Per-launch DRAM bytes of `kernel_name` from the committed ncu summary, if any."""
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        d = json.load(open(path))
        return d.get(kernel_name)
    except Exception:
        return None


# ---------------------------------------------------------------- CPU baseline (oracle)
def _oracle_sample(name: str):
    from workloads import programs, data
    if name in ("weather", "weak", "weather_small"):
        desc = programs.weather(n=(64, 64, 128))
        return desc, data.weather_inputs(desc, 3), "weather program on a 64x64x128 sub-grid"
    if name == "tiny":
        desc = programs.tiny()
        return desc, data.uniform(desc, 1), "tiny 32^3"
    if name == "fig3":
        desc = programs.fig3(n=(64, 64, 128))
        return desc, data.fig3_inputs(desc, 3), "fig3 on 64x64x128"
    if name == "suite":
        desc = programs.gen_suite(seed=0, n=(64, 64, 64))
        return desc, data.uniform(desc, 3), "suite program on 64^3"
    desc = programs.stress(m=2, n=(64, 64, 64))
    return desc, data.uniform(desc, 5), "stress 2 fields on 64^3"


def _oracle_worker(args):
    name, budget_s = args
    from oracle import interp
    desc, inp, _ = _oracle_sample(name)
    t0 = time.perf_counter()
    steps = 0
    while True:
        inp = interp.run(desc, inp, 1)
        steps += 1
        if time.perf_counter() - t0 > budget_s:
            break
    return desc.npts * steps, time.perf_counter() - t0


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def cpu_baseline(name: str, budget_s: float = 8.0):
    """The oracle (numpy, unfused, as it stands) on bounded samples of the same workload: one
    process on one core, then one process per host core (each on its own sub-grid, capped at 64)."""
    import multiprocessing as mp
    pts, dt = _oracle_worker((name, budget_s))
    _, _, sample = _oracle_sample(name)
    one = pts / dt
    ncores = min(os.cpu_count() or 1, 64)
    allc = None
    if ncores > 1:
        try:
            ctx = mp.get_context("fork")
            t0 = time.perf_counter()
            with ctx.Pool(ncores) as pool:
                res = pool.map(_oracle_worker, [(name, budget_s)] * ncores)
            wall = time.perf_counter() - t0
            allc = {"value": sum(r[0] for r in res) / wall, "cores": ncores, "wall_s": round(wall, 2)}
        except Exception as e:   # reported, never guessed
            allc = {"error": f"{type(e).__name__}: {e}"}
    return {"value": one, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"{sample}, numpy oracle unfused, 1 step per timing, {budget_s:.0f} s budget per process",
            "all_cores": allc, "host_cpu": cpu_model(), "host_cores": os.cpu_count()}


# ---------------------------------------------------------------- GPU timing
AUTOTUNE_CANDIDATES = [  # (tile, stages, zunroll, ringunroll, minblocks, canvas_ld[, pblock x, pair_zq[, inline_xy]])
    ((32, 8, 64), 2, 1, 0, 0, 1), ((32, 8, 64), 2, 1, 0, -1, 1), ((32, 8, 64), 2, 1, 0, -1, 0), ((32, 8, 64), 2, 1, 0, 0, 0),
    ((32, 8, 32), 2, 1, 0, -1, 1), ((32, 8, 32), 2, 1, 0, 0, 0), ((32, 8, 0), 2, 1, 0, -1, 1), ((64, 4, 64), 2, 1, 0, 0, 1),
    ((32, 8, 64), 3, 1, 0, -1, 1), ((32, 8, 64), 2, 1, 1, -1, 1),
    ((64, 8, 64), 2, 2, 0, 0, 1),   # z-unroll 2 on 64x8: the fastest for the fp32 suite groups (tools/ab.py)
    # canvas pairs (two x-adjacent points per thread, 16-byte vector shared loads/stores), with and
    # without z-column register queues
    ((32, 8, 32), 2, 1, 0, -1, 1, 2, 0), ((32, 8, 64), 2, 1, 0, -1, 1, 2, 0), ((32, 8, 64), 2, 1, 0, -1, 1, 2, 1),
    ((32, 8, 64), 2, 1, 0, -1, 0, 2, 1), ((32, 8, 64), 2, 1, 0, 0, 1, 2, 1), ((32, 8, 32), 2, 1, 0, -1, 1, 2, 1),
    # z chunks of 43 planes: 3 chunks of a 128-plane column, 6.9 waves of 3 CTAs/SM instead of 4.6
    # (wave quantisation; measured -2..-4 % on the flux groups)
    ((32, 8, 43), 2, 1, 0, -1, 1, 2, 1), ((32, 8, 43), 2, 1, 0, -1, 1, 2, 0), ((32, 8, 43), 2, 1, 0, -1, 1),
    # in-group values at xy offsets from shared memory instead of recomputed by their readers
    ((32, 8, 43), 2, 1, 0, -1, 1, 2, 1, 0), ((32, 8, 32), 2, 1, 0, -1, 1, 2, 0, 0),
    # taller / wider pair tiles: less halo per point (36x20/512 = 1.41 vs 36x12/256 = 1.69 box/tile)
    ((32, 16, 43), 2, 1, 0, -1, 1, 2, 1), ((32, 16, 43), 2, 1, 0, -1, 1, 2, 0), ((64, 8, 43), 2, 1, 0, -1, 1, 2, 1),
    # three TMA stages for pairs: ncu showed 12 % of the flux group's warp samples waiting on the
    # mbarrier of the current plane (one plane of prefetch is not enough latency cover)
    ((32, 8, 43), 3, 1, 0, -1, 1, 2, 1), ((32, 8, 43), 3, 1, 0, -1, 1, 2, 0), ((32, 8, 64), 3, 1, 0, -1, 1, 2, 1),
    # shorter / taller pair tiles: smaller planes make room for a third stage (4 rows), or less halo (12)
    ((32, 4, 43), 3, 1, 0, -1, 1, 2, 1), ((32, 4, 43), 2, 1, 0, -1, 1, 2, 1), ((32, 12, 43), 2, 1, 0, -1, 1, 2, 1)]


def cand_kw(base_kw, c):
    kw = dict(base_kw)
    kw.update(tile=tuple(c[0]), stages=c[1], zunroll=c[2], ringunroll=c[3], minblocks=c[4] if len(c) > 4 else 0,
              canvas_ld=c[5] if len(c) > 5 else 1, pblock=(c[6] if len(c) > 6 else 1, 1),
              pair_zq=c[7] if len(c) > 7 else 1, inline_xy=c[8] if len(c) > 8 else 1)
    return kw


def cand_norm(c):
    """Full 9-field form [tile, stages, zunroll, ringunroll, minblocks, canvas_ld, pblock_x, pair_zq, inline_xy]."""
    full = list(c) + [None] * (9 - len(c))
    dflt = [None, 2, 1, 0, 0, 1, 1, 1, 1]
    return [list(full[0])] + [full[i] if full[i] is not None else dflt[i] for i in range(1, 9)]


def autotune(prog, plan, dev, base_kw, steps=6):
    """Per-group launch configuration: run the whole plan under each candidate (tile, stages,
    zunroll, ...) with per-group CUDA-event timing and keep, for every group, its fastest legal
    candidate.  Mutates the arrays (they are synthetic; the timed runs start from the result)."""
    import torch
    import paper_conf_sc_wahibm14_b200 as kf
    best = None
    tried = []
    for cand in AUTOTUNE_CANDIDATES:
        kw = cand_kw(base_kw, cand)
        try:
            ex = kf.Exec(prog, plan, kf.Target(**kw))
        except Exception:
            continue
        sb = ex.scratch_bytes()
        scr = torch.empty(sb, dtype=torch.uint8, device="cuda") if sb else None
        ex.run(dev, scr, 2)
        torch.cuda.synchronize()
        ex.set_profiling(True)
        ex.run(dev, scr, steps)
        torch.cuda.synchronize()
        gms, _ = ex.group_times()
        tried.append((tuple(cand), [g / steps for g in gms]))
        if best is None:
            best = [(g / steps, kw, cand) for g in gms]
        else:
            best = [min(b, (g / steps, kw, cand), key=lambda v: v[0]) for b, g in zip(best, gms)]
        del ex, scr
    return [kf.Target(**kw) for _, kw, _ in best], [cand_norm(c) for _, _, c in best], tried


def max_over_ranks(x: float) -> float:
    import torch
    if torch.distributed.is_initialized():
        t = torch.tensor([x], dtype=torch.float64, device="cuda")
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        return float(t.item())
    return x


class Runner:
    """One rank's view of the hot path: a kf.Exec (1 GPU) or a kf.Dist over NCCL (N GPUs)."""

    def __init__(self, prog, plan, target, group_targets, dist_info):
        import torch
        import paper_conf_sc_wahibm14_b200 as kf
        self.ex = kf.Exec(prog, plan, target, group_targets=group_targets)
        sb = self.ex.scratch_bytes()
        self.scratch = torch.empty(sb, dtype=torch.uint8, device="cuda") if sb else None
        self.dist = None
        if dist_info is not None:
            px, py, rank, world, nid = dist_info
            self.dist = kf.Dist([self.ex], px, py, rank, world, nid)

    def run(self, dev, nsteps, stream):
        if self.dist is None:
            self.ex.run(dev, self.scratch, nsteps, stream=stream)
        else:
            self.dist.run([dev], [self.scratch], nsteps, stream=stream)


def time_runner(rn, dev, steps, warmup, stream, profile=False, clk=None):
    import torch
    rn.run(dev, warmup, stream)
    torch.cuda.synchronize()
    if profile:
        rn.ex.set_profiling(True)
    if torch.distributed.is_initialized():
        torch.distributed.barrier()
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    if clk is not None:
        clk.mark_start()
    e0.record(stream)
    rn.run(dev, steps, stream)
    e1.record(stream)
    torch.cuda.synchronize()
    if clk is not None:
        clk.mark_end()
    ms = e0.elapsed_time(e1)
    gt = None
    if profile:
        gt = rn.ex.group_times()
        rn.ex.set_profiling(False)
    return ms, gt


def parity_windows(wl, prog, rn, rank, world, stream, nsteps=2, w=8):
    """Parity of the configuration just timed: fresh seeded inputs, `nsteps` steps through the same
    executor (plan and per-group launch configurations), then windows compared with the oracle on
    dependency-cone crops (oracle/windows.py).  N = 1: windows anywhere (periodic seams, corners,
    tile edges); N > 1: windows deep inside the rank's sub-domain (the cone stays local)."""
    import numpy as np
    import torch
    from oracle import graph, interp
    from oracle.windows import crop, crop_window, dependency_radius
    desc = wl.desc
    if wl.gen not in ("weather", "uniform", "fig3", "device_uniform", "weather_tiled"):
        return {"skipped": f"inputs of workload {wl.name} are not reproducible on the host"}
    M = dependency_radius(desc, nsteps) + 1
    nx, ny, _ = desc.n
    if world == 1:
        pos = [(0, 0), (nx - 4, 3), (nx // 2 - 4, ny - 5), (131 % nx, 257 % ny), (nx - w, ny - w), (64 % nx, 64 % ny)]
    else:
        pos = [(M + 1, M + 1), (nx // 2, ny // 2), (nx - M - w - 1, ny - M - w - 1)]
    dev, host_in = wl.inputs(prog, rank)
    L = prog.layout()
    g = desc.ghost
    nz2 = desc.n[2] + 2 * g[2]

    def dev_cols(x0, wd, mg):   # kf-layout columns / rows of a wrapped window (+ margin and ghosts)
        xi = (np.arange(-mg - g[0], wd + mg + g[0]) + x0) % nx + g[0]
        return torch.as_tensor(L.xoff - g[0] + xi, device="cuda")

    def dev_rows(y0, wd, mg):
        return torch.as_tensor((np.arange(-mg - g[1], wd + mg + g[1]) + y0) % ny + g[1], device="cuda")

    crops = None
    if host_in is None:   # device-generated inputs (stress, weak): the crops' inputs read from the device
        crops = []
        for (x0, y0) in pos:
            ci, ri = dev_cols(x0, w, M), dev_rows(y0, w, M)
            sub = desc.with_(n=(w + 2 * M, w + 2 * M, desc.n[2]), bc=(0, 0, desc.bc[2]))
            sin = {nm: t.view(nz2, L.rows, L.pitch)[:, ri][:, :, ci].cpu().numpy() for (nm, _), t in zip(desc.arrays, dev)}
            crops.append((sub, sin))
    rn.run(dev, nsteps, stream)
    torch.cuda.synchronize()
    names = [nm for x, (nm, _) in enumerate(desc.arrays)
             if not graph.writers(desc, x) or graph.step_live(desc, x)]
    wins = {}
    for (x0, y0) in pos:   # the run's windows (interior planes), read from the device
        ci, ri = dev_cols(x0, w, 0)[g[0]:g[0] + w], dev_rows(y0, w, 0)[g[1]:g[1] + w]
        for (nm, _), t in zip(desc.arrays, dev):
            if nm in names:
                wins[(nm, x0, y0)] = t.view(nz2, L.rows, L.pitch)[g[2]:g[2] + desc.n[2]][:, ri][:, :, ci].cpu().numpy()
    del dev
    t0 = time.perf_counter()
    ok, bad = 0, []
    for i, (x0, y0) in enumerate(pos):
        sub, sin = crop(desc, host_in, x0, y0, w, M) if crops is None else crops[i]
        ref = interp.run(sub, sin, nsteps)
        for nm in names:
            r = crop_window(sub, ref[nm], w, M)
            g_ = wins[(nm, x0, y0)]
            bt = np.uint32 if r.dtype == np.float32 else np.uint64
            if np.array_equal(g_.view(bt), r.view(bt)):
                ok += 1
            else:
                bad.append([nm, x0, y0])
    return {"windows": len(pos), "window": f"{w}x{w}x{desc.n[2]}", "steps": nsteps, "arrays": names,
            "compared": ok + len(bad), "bit_exact": not bad, "mismatches": bad[:8], "margin": M,
            "oracle_s": round(time.perf_counter() - t0, 2),
            "method": "oracle/windows.py dependency-cone crops of fresh seeded inputs (device-generated ones read back "
                      "from the device), same executor as timed"}


def run_kf(args):
    import numpy as np
    import torch
    import paper_conf_sc_wahibm14_b200 as kf
    from workloads.program import PROG_RELAX_ALL

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        raise SystemExit(f"bench.py: WORLD_SIZE={world} but --gpus {args.gpus}")
    if world > 1:
        torch.cuda.set_device(local)
        torch.distributed.init_process_group("nccl", device_id=torch.device("cuda", local))
    else:
        torch.cuda.set_device(0)
    wl = Workload(args.workload, world)
    desc = wl.desc
    if args.relax_all and desc.name == "weather":
        desc = wl.desc = desc.with_(flags=PROG_RELAX_ALL)
    S = max(1, args.unroll)
    if S > 1:   # NEXT-4: S timesteps as one step of the unrolled program (plans may fuse across steps)
        from workloads import programs
        from workloads.program import unroll
        if desc.name == "weather":   # cross-step fusion accumulates halos: a deeper periodic ghost (V6)
            desc = programs.weather(n=desc.n, ghost=(2 * S, 2 * S, 2), relax=desc.flags)
        desc = wl.desc = unroll(desc, S)
        wl.label += f", unrolled x{S} (temporal fusion: one step = {S} timesteps)"
    tkw = dict(wl.tkw)
    if args.tile:
        tkw["tile"] = tuple(int(v) for v in args.tile.split(","))
    if args.stages:
        tkw["stages"] = args.stages
    if args.threads:
        tkw["threads"] = args.threads
    # single domain: periodic ghost fills between groups (default; measured faster than ghost copies
    # written by the producing groups' epilogues, profiles/round2_summary.md), or --ghostwrite;
    # decomposed: halo exchanges replace the fills
    tkw["ghostwrite"] = 1 if (world == 1 and args.ghostwrite) else 0
    if world > 1:
        px, py = grid_for(world)
        tkw["internal_axes"] = (1 if px > 1 else 0) | (2 if py > 1 else 0)
    target = kf.Target(**tkw)
    prog = kf.Program(desc)          # the per-GPU sub-domain program
    committed = None
    if args.plan == "auto":
        # the committed configuration of config 3: plan and per-group launch configurations chosen by
        # measured selection + per-group autotuning on B200 in an earlier run (source recorded in the
        # file), replayed as is -- reproducible, and the ncu evidence under profiles/ names its kernels
        path = os.path.join(ROOT, "profiles", "bench_timed_config.json")
        if (args.workload == "weather" and S == 1 and not args.relax_all and not args.tuned and world == 1
                and not args.ghostwrite and os.path.exists(path)):
            committed = json.load(open(path))
            if committed.get("ghostwrite", 0) != tkw["ghostwrite"]:
                committed = None
        if committed is None:
            args.plan = "select"
    if committed is not None:
        plan = committed["plan_labels"]
        plan_kind = f"committed tuned configuration (profiles/bench_timed_config.json; {committed.get('source', '')})"
        args.tuned = json.dumps(committed["per_group_launch_config"])
    else:
        plan, plan_kind = (None, None) if args.plan == "select" else choose_plan(prog, target, args.plan)

    def new_dist_info():
        """A fresh NCCL unique id (broadcast from rank 0) for every communicator kf.Dist creates."""
        if world == 1:
            return None
        px, py = grid_for(world)
        nid = kf.dist_unique_id() if rank == 0 else bytes(128)
        t = torch.tensor(list(nid), dtype=torch.uint8, device="cuda")
        torch.distributed.broadcast(t, 0)
        return (px, py, rank, world, bytes(t.cpu().tolist()))
    dev, _ = wl.inputs(prog, rank)
    stream = torch.cuda.current_stream()
    t0 = time.time()
    candidates, ranked = None, []
    if plan is None:   # measured plan selection (rank 0 decides, every rank runs the same plan)
        if rank == 0:
            plan, plan_kind, candidates, ranked = select_plan(prog, target, dev)
        if world > 1:
            obj = [(plan, plan_kind, candidates)]
            torch.distributed.broadcast_object_list(obj, 0)
            plan, plan_kind, candidates = obj[0]
    tuned, gtargets, tried = None, None, None
    if args.tuned:   # fixed per-group configs (e.g. for an ncu run of exactly the timed configuration)
        tuned = json.loads(args.tuned)
        gtargets = [kf.Target(**cand_kw(tkw, c)) for c in tuned]
    elif args.autotune:
        if rank == 0:
            gtargets, tuned, tried = autotune(prog, plan, dev, tkw)
            # the runner-up of the measured selection, autotuned too: the per-group launch
            # configurations can reorder close plans (sum of the per-group best times decides)
            if args.plan == "select" and len(ranked) > 1 and ranked[0][0] == plan:
                alt, alt_kind = ranked[1]
                g2, t2, tr2 = autotune(prog, alt, dev, tkw)
                est = lambda tr: sum(min(g[i] for _, g in tr) for i in range(len(tr[0][1])))   # noqa: E731
                if tr2 and tried and est(tr2) < est(tried):
                    plan, plan_kind = alt, alt_kind + " (runner-up of the measured candidates, faster once autotuned)"
                    gtargets, tuned, tried = g2, t2, tr2
        if world > 1:
            obj = [tuned]
            torch.distributed.broadcast_object_list(obj, 0)
            tuned = obj[0]
            gtargets = [kf.Target(**cand_kw(tkw, c)) for c in tuned]
    rn = Runner(prog, plan, target, gtargets, new_dist_info())
    jit_s = time.time() - t0
    info = rn.ex.info()

    with ClockSampler(local) as clk:
        ms, _ = time_runner(rn, dev, args.steps, args.warmup, stream, clk=clk)
    ms = max_over_ranks(ms)
    clocks = clk.summary()
    # per-group device times over a second timed region (events on the launch stream)
    ms_prof, (gms, nlaunch) = time_runner(rn, dev, args.steps, 1, stream, profile=True)
    # sustained rate: a longer region (the flux groups slow down once the board reaches its power limit)
    sus_steps = max(200, args.steps)
    ms_sus, _ = time_runner(rn, dev, sus_steps, 1, stream)
    ms_sus = max_over_ranks(ms_sus)
    # unfused plan on the same inputs: speedup vs unfused, and the original per-kernel times
    unf = None
    k_ms = None
    if not args.no_unfused and args.plan != "unfused":
        ut = kf.Target(**dict(tkw))
        rn_u = Runner(prog, list(range(prog.nk)), ut, None, new_dist_info())
        ms_u, _ = time_runner(rn_u, dev, args.steps, args.warmup, stream)
        ms_u = max_over_ranks(ms_u)
        _, (kms, _) = time_runner(rn_u, dev, args.steps, 1, stream, profile=True)
        k_ms = [v / args.steps for v in kms]
        unf = {"ms_per_step": ms_u / args.steps, "bytes_per_step": rn_u.ex.info().compulsory_bytes_per_step,
               "launches_per_step": rn_u.ex.info().launches_per_step}
        del rn_u
    # end-to-end through the public API with host buffers (copies inside the timed region)
    e2e = None
    if not args.no_e2e and wl.gen not in ("device_uniform", "weather_tiled"):
        k = max(1, min(args.steps, 3))
        if rn.dist is None:
            host = [t.cpu().pin_memory() for t in dev]
            rn.ex.run_host([h.data_ptr() for h in host], 1, stream=stream.cuda_stream)   # warm (allocs, full upload)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            h2d = d2h = 0
            for _ in range(k):
                h2d, d2h = rn.ex.run_host([h.data_ptr() for h in host], 1, stream=stream.cuda_stream)
            dt = time.perf_counter() - t0
            how = "kf_run_host (C ABI, pinned host buffers), host wall clock, synchronising"
        else:
            ins = [x for x in range(len(desc.arrays)) if prog.array_info(x).upward_exposed]
            outs = [x for x in range(len(desc.arrays)) if prog.array_info(x).step_live]
            host = {x: dev[x].cpu().pin_memory() for x in set(ins) | set(outs)}
            torch.cuda.synchronize()
            torch.distributed.barrier()
            t0 = time.perf_counter()
            for _ in range(k):
                for x in ins:
                    dev[x].copy_(host[x], non_blocking=True)
                rn.run(dev, 1, stream)
                for x in outs:
                    host[x].copy_(dev[x], non_blocking=True)
                torch.cuda.synchronize()
            dt = time.perf_counter() - t0
            h2d = sum(host[x].numel() * host[x].element_size() for x in ins)
            d2h = sum(host[x].numel() * host[x].element_size() for x in outs)
            how = "kf.Dist.run with pinned host buffers copied in/out every step, host wall clock"
        dt = max_over_ranks(dt)
        e2e = {"value": wl.global_npts * k * S / dt, "unit": UNIT, "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
               "steps": k, "timing": how + ", max over ranks"}
        del host

    bytes_step = info.compulsory_bytes_per_step
    value = wl.global_npts * args.steps * S / (ms / 1e3)
    peaks = measured_peaks()
    hbm_peak = peaks["hbm_gbs"] if peaks and "hbm_gbs" in peaks else 6650.0
    peak_src = "MEASURED_PEAKS.json hbm_gbs (burst copy)" if peaks else "B200_PROFILING.md fallback 6.65 TB/s"
    g_dom = int(np.argmax(gms))
    gi = rn.ex.group_info(g_dom)
    gname = gi.name.decode() if isinstance(gi.name, bytes) else gi.name
    t_launch_ms = gms[g_dom] / args.steps
    achieved = gi.bytes_per_launch / (t_launch_ms / 1e3) / 1e9
    roofline = {"bound": "hbm", "achieved": achieved, "peak": hbm_peak, "unit": "GB/s", "frac": achieved / hbm_peak,
                "traffic": ncu_traffic(gname), "kernel": gname, "peak_source": peak_src,
                "share_of_step": gms[g_dom] / max(1e-9, sum(gms)),
                "algorithmic_bytes_per_launch": gi.bytes_per_launch,
                "per_group_ms_per_step": [g / args.steps for g in gms]}
    # on-chip roofline of the same kernel: its canvas shared-memory traffic (loads + stores + TMA
    # writes per fast iteration, from the lowering) over the SMEM bandwidth (128 B/clk/SM at the
    # measured SM clock) -- the bound of groups whose halo recompute outweighs their HBM bytes
    sm_clk = (clocks.get("sm_mhz") or 1965) * 1e6
    onchip = {"bound": "smem", "achieved": gi.onchip_bytes_per_launch / (t_launch_ms / 1e3) / 1e9,
              "peak": 128 * 148 * sm_clk / 1e9, "unit": "GB/s",
              "algorithmic_bytes_per_launch": gi.onchip_bytes_per_launch,
              "peak_source": "128 B/clk/SM x 148 SMs x SM clock (B300_MICROARCH / B200_PROFILING)"}
    onchip["frac"] = onchip["achieved"] / onchip["peak"]
    roofline["onchip"] = onchip
    achieved_step = bytes_step / (ms / args.steps / 1e3) / 1e9
    # NEXT-2 (Figs. 6-8 analogue): per group measured vs projected vs the original kernels' sum
    per_groups = []
    canon = []
    m_ = {}
    for g in plan:
        canon.append(m_.setdefault(g, len(m_)))
    tgt_of = gtargets if gtargets else [target] * len(gms)
    for g in range(len(gms)):
        per_g, _, _ = prog.project(plan, tgt_of[g])
        gi_ = rn.ex.group_info(g)
        ks = [k for k in range(prog.nk) if canon[k] == g]
        row = {"group": g, "kernel": gi_.name.decode() if isinstance(gi_.name, bytes) else gi_.name,
               "kernels": len(ks), "measured_ms": gms[g] / args.steps,
               "t_model_ms": per_g[g].t_model_s * 1e3,
               "t_bytes_ms": (per_g[g].bytes_read + per_g[g].bytes_written) / (hbm_peak * 1e9) * 1e3,
               "original_sum_ms": sum(k_ms[k] for k in ks) if k_ms else None,
               "regs": gi_.regs, "regs_est": per_g[g].regs_est, "smem": gi_.smem_bytes,
               "threads": gi_.threads, "frac_of_copy_peak": gi_.bytes_per_launch / (gms[g] / args.steps / 1e3) / 1e9 / hbm_peak}
        per_groups.append(row)
    mod_err = [abs(r["t_model_ms"] / r["measured_ms"] - 1) for r in per_groups if r["measured_ms"] > 0]
    per, _, t_proj = prog.project(plan, target)
    parity = None
    if not args.no_parity:
        parity = parity_windows(wl, prog, rn, rank, world, stream)
        if world > 1:
            obj = [parity]
            allp = [None] * world
            torch.distributed.all_gather_object(allp, parity)
            parity = {"ranks": allp, "bit_exact": all(p_.get("bit_exact", False) for p_ in allp if "skipped" not in p_)}
    px, py = grid_for(world)
    res = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": ms / args.steps / S, "higher_is_better": True, "scaling": wl.scaling, "vs_baseline": None,
        "dtype": "f64" if desc.dtype == 1 else "f32", "data": "synthetic (seeded, paper-shaped fields)",
        "config": {"workload": wl.label + (" with RELAX_ALL renaming" if desc.flags & 2 else ""),
                   "plan": f"{plan_kind}: {info.n_groups} fused groups of {prog.nk} kernels",
                   "plan_labels": plan, "tile": list(target.tile), "stages": target.stages,
                   "threads": target.threads, "ghostwrite": tkw["ghostwrite"],
                   "l2": "inputs larger than L2 (each array > 126 MB), no flush" if desc.npts * desc.es > 126e6
                   else "inputs smaller than L2 (no flush; small config)",
                   "parallelism": (f"xy domain decomposition {px}x{py}, NCCL halo exchange (batched per phase, "
                                   f"overlapped with interior tiles, CUDA graph), {wl.scaling}") if world > 1 else "1 GPU",
                   "local_grid": list(desc.n), "global_points": wl.global_npts,
                   "graph": True, "jit_s": round(jit_s, 2),
                   "per_group_launch_config": [cand_norm(c) for c in tuned] if tuned else "uniform",
                   "plan_candidates": candidates,
                   "autotune_tried": [{"config": list(c), "group_ms": [round(x, 4) for x in g]} for c, g in tried]
                   if tried else None},
        "hbm_gbs_compulsory": achieved_step,
        "frac_of_measured_copy": achieved_step / hbm_peak,
        "frac_of_nominal_8TBs": achieved_step / 8000.0,
        "compulsory_bytes_per_step": bytes_step,
        "fills_per_step": info.fills_per_step,
        "projected_ms_per_step": t_proj * 1e3,
        "model_ms_per_step": sum(g.t_model_s for g in per) * 1e3,
        "sustained": {"steps": sus_steps, "ms_per_step": ms_sus / sus_steps / S,
                      "value": wl.global_npts * sus_steps * S / (ms_sus / 1e3)},
        "per_group": per_groups,
        "model_error_max": max(mod_err) if mod_err else None,
        "roofline": roofline,
        "parity": parity,
        "gpu_launches": int(info.launches_per_step * args.steps),
        "clocks": clocks,
    }
    if unf:
        res["unfused"] = unf
        res["speedup_vs_unfused"] = unf["ms_per_step"] / (ms / args.steps)
        traffic_ratio = bytes_step / unf["bytes_per_step"]
        time_ratio = (ms / args.steps) / unf["ms_per_step"]
        res["fusion_efficiency"] = traffic_ratio / time_ratio        # Eq. 12
    if e2e:
        res["e2e"] = e2e
    if rank == 0 and not args.no_cpu:
        res["cpu_baseline"] = cpu_baseline(args.workload)
    if rank == 0:
        print(json.dumps(res))
    if world > 1:
        torch.distributed.barrier()
        torch.distributed.destroy_process_group()


def run_all_plans(args):
    """Config 2: every legal plan of the suite program at 256^3 timed on one GPU
    (JIT of all plans on parallel host threads, identical groups compiled once), reporting the
    best, the worst, the unfused plan and Fusion Efficiency; one JSON line with every plan."""
    import torch
    from concurrent.futures import ThreadPoolExecutor
    import paper_conf_sc_wahibm14_b200 as kf
    torch.cuda.set_device(0)
    wl = Workload(args.workload, 1)
    tkw = dict(wl.tkw, ghostwrite=0)
    target = kf.Target(**tkw)
    prog = kf.Program(wl.desc)
    plans = prog.legal_plans(target)
    dev, _ = wl.inputs(prog, 0)
    t0 = time.time()
    with ThreadPoolExecutor(max_workers=min(32, os.cpu_count() or 4)) as pool:
        execs = list(pool.map(lambda pl: kf.Exec(prog, pl, target), plans))
    jit_s = time.time() - t0
    rows = []
    for pl, ex in zip(plans, execs):
        ms = time_exec(ex, dev, args.steps, warm=args.warmup)
        b = ex.info().compulsory_bytes_per_step
        rows.append({"plan": pl, "groups": len(set(pl)), "ms_per_step": ms, "bytes_per_step": b,
                     "proj_ms": prog.project(pl, target)[2] * 1e3})
    del execs
    unf = [r for r in rows if r["groups"] == prog.nk][0]
    best = min(rows, key=lambda r: r["ms_per_step"])
    worst = max(rows, key=lambda r: r["ms_per_step"])
    fe = lambda r: (r["bytes_per_step"] / unf["bytes_per_step"]) / (r["ms_per_step"] / unf["ms_per_step"])  # noqa: E731
    npts = wl.desc.npts
    out = {"metric": METRIC, "value": npts / (best["ms_per_step"] / 1e3), "unit": UNIT, "n_gpus": 1,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": best["ms_per_step"], "higher_is_better": True,
           "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
           "config": {"workload": wl.label, "mode": "every legal plan timed (P:435, P:481)", "legal_plans": len(rows),
                      "tile": list(target.tile), "jit_s": round(jit_s, 1)},
           "best": dict(best, fusion_efficiency=fe(best), speedup_vs_unfused=unf["ms_per_step"] / best["ms_per_step"]),
           "worst": dict(worst, fusion_efficiency=fe(worst), speedup_vs_unfused=unf["ms_per_step"] / worst["ms_per_step"]),
           "unfused": unf,
           "projection_rank_corr": None,
           "plans": rows}
    try:
        import numpy as np
        a = np.argsort(np.argsort([r["proj_ms"] for r in rows]))
        b = np.argsort(np.argsort([r["ms_per_step"] for r in rows]))
        out["projection_rank_corr"] = float(np.corrcoef(a, b)[0, 1])
    except Exception:
        pass
    print(json.dumps(out))


def run_reference(args):
    """--impl reference: the oracle as it stands on the host cores (rank 0 only), a bounded
    sub-grid sample of the same workload per timed step."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    from oracle import interp
    desc, inp, sample = _oracle_sample(args.workload)
    wl_label = Workload(args.workload, 1).label if args.workload != "stress" else "config 5 stress"
    for _ in range(args.warmup):
        inp = interp.run(desc, inp, 1)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        inp = interp.run(desc, inp, 1)
    dt = time.perf_counter() - t0
    value = desc.npts * args.steps / dt
    res = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": int(os.environ.get("WORLD_SIZE", "1")),
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3,
           "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
           "dtype": "f64" if desc.dtype == 1 else "f32", "data": "synthetic", "impl": "reference",
           "config": {"workload": wl_label},
           "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle",
                            "sample": sample + ", 1 step per timed step (numpy oracle, unfused)"},
           "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(res))


def relaunch_distributed(n: int) -> int:
    """--gpus N > 1 without a launcher: one rank per GPU under torch.distributed.run."""
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="kf", choices=["kf", "reference"])
    ap.add_argument("--workload", default="weather")
    ap.add_argument("--plan", default="auto",
                    help="auto: config 3 replays the committed tuned configuration (profiles/bench_timed_config.json), "
                         "other workloads select; select: measured choice among the searches' candidates + autotune; "
                         "best: HGGA/brute on projected time; unfused; hand; or a JSON label list")
    ap.add_argument("--relax-all", type=int, default=0, help="weather: rename every written array (KF_PROG_RELAX_ALL)")
    ap.add_argument("--unroll", type=int, default=1, help="NEXT-4 temporal fusion: plan over S timesteps as one step")
    ap.add_argument("--tile", default=None)
    ap.add_argument("--stages", type=int, default=None)
    ap.add_argument("--threads", type=int, default=None)
    ap.add_argument("--ghostwrite", action="store_true", help="ghost copies written by the producing groups "
                                                                  "instead of ghost-fill launches (A/B)")
    ap.add_argument("--all-plans", action="store_true", help="time every legal plan (programs of <= 14 kernels)")
    ap.add_argument("--no-unfused", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-parity", action="store_true")
    ap.add_argument("--autotune", type=int, default=1, help="per-group launch configuration by measurement (1/0)")
    ap.add_argument("--tuned", default=None, help="JSON per-group configs as printed in config.per_group_launch_config: "
                                                  "[tile, stages, zunroll, ringunroll, minblocks, canvas_ld, pblock_x, pair_zq[, inline_xy]]")
    args = ap.parse_args()
    if args.warmup < 3 and args.impl == "kf":
        args.warmup = 3
    if args.impl == "reference":
        run_reference(args)
        return
    if args.gpus < 1:
        raise SystemExit("--gpus must be >= 1")
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        import torch
        have = torch.cuda.device_count()
        if have < args.gpus:
            raise SystemExit(f"bench.py: --gpus {args.gpus} but only {have} CUDA device(s) visible")
        sys.exit(relaunch_distributed(args.gpus))
    if args.all_plans:
        run_all_plans(args)
    else:
        run_kf(args)


if __name__ == "__main__":
    main()
