"""NEXT-3: test-suite sweep over Table V ranges with Fig. 9-style speedups.

For every (kernels, arrays) pair the suite generator (workloads.programs.gen_suite)
builds a program with average thread load `--load` (Table V: 4..12; Fig. 9 uses 8).  Each program
runs unfused (singleton groups) and under the plans the searches propose (HGGA on the projected time
and on compulsory bytes); every plan is timed with CUDA events after warm-up, with single
canvas points and with canvas pairs (the faster is kept, for the unfused baseline too).  One JSON
line per benchmark: speedup of the fastest fused plan over unfused, Fusion Efficiency (Eq. 12,
P:501), projected vs measured time, compulsory bytes.

  python tools/suite_sweep.py [--kernels 10,20,...] [--ratios 1,2] [--load 8] [--n 512,512,64]
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def time_plan(kf, prog, plan, dev, target, steps):
    import torch
    ex = kf.Exec(prog, plan, target)
    sb = ex.scratch_bytes()
    scr = torch.empty(sb, dtype=torch.uint8, device="cuda") if sb else None
    ex.run(dev, scr, 2)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    ex.run(dev, scr, steps)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / steps
    info = ex.info()
    return ms, info.compulsory_bytes_per_step, info.n_groups


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--kernels", default="10,20,40,60,80,100")
    ap.add_argument("--ratios", default="1,2", help="arrays per kernel (Table V: 20..200 arrays for 10..100 kernels)")
    ap.add_argument("--load", type=int, default=8)
    ap.add_argument("--n", default="512,512,64")
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--seed", type=int, default=1)
    args = ap.parse_args()
    import torch
    import paper_conf_sc_wahibm14_b200 as kf
    from workloads import programs as P
    n = tuple(int(v) for v in args.n.split(","))
    # launch configurations tried for every plan (the fastest is kept): single canvas points and
    # canvas pairs (two x-adjacent points per thread, vector shared loads)
    targets = [kf.Target(tile=(32, 8, 64)), kf.Target(tile=(32, 8, 64), pblock=(2, 1))]
    target = targets[0]

    def best_time(prog, plan, dev):
        best = None
        for t in targets:
            try:
                r = time_plan(kf, prog, plan, dev, t, args.steps)
            except Exception:   # noqa: BLE001 -- a configuration illegal for this plan (V7/V8)
                continue
            if best is None or r[0] < best[0]:
                best = r
        if best is None:
            raise RuntimeError("no legal launch configuration")
        return best
    for nk in [int(v) for v in args.kernels.split(",")]:
        for na in [int(float(r) * nk) for r in args.ratios.split(",")]:
            t0 = time.time()
            try:
                desc = P.gen_suite(n_kernels=nk, n_arrays=na, seed=args.seed, n=n, load=args.load, max_tries=2000)
            except RuntimeError as e:
                print(json.dumps({"kernels": nk, "arrays": na, "error": str(e)}), flush=True)
                continue
            prog = kf.Program(desc)
            L = prog.layout()
            g = torch.Generator(device="cuda").manual_seed(args.seed)
            dev = [torch.rand(L.elems, generator=g, device="cuda", dtype=torch.float32) * 2 - 1 for _ in desc.arrays]
            ms_u, b_u, _ = best_time(prog, list(range(nk)), dev)
            res = []
            for name, method in (("hgga_time", kf.SEARCH_HGGA), ("hgga_bytes", kf.SEARCH_HGGA_BYTES)):
                plan, _ = prog.search(method, target, seed=1)
                per, _, t_proj = prog.project(plan, target)
                try:
                    ms, b, m = best_time(prog, plan, dev)
                except Exception as e:   # noqa: BLE001 -- report and continue the sweep
                    res.append({"plan": name, "error": str(e)[:160]})
                    continue
                res.append({"plan": name, "groups": m, "ms": round(ms, 4), "bytes": b,
                            "projected_ms": round(t_proj * 1e3, 4),
                            "model_ms": round(sum(p.t_model_s for p in per) * 1e3, 4)})
            ok = [r for r in res if "ms" in r]
            best = min(ok, key=lambda r: r["ms"]) if ok else None
            out = {"kernels": nk, "arrays": na, "load": args.load, "grid": list(n), "dtype": "f32",
                   "unfused_ms": round(ms_u, 4), "unfused_bytes": b_u, "plans": res, "wall_s": round(time.time() - t0, 1)}
            if best:
                out["speedup"] = round(ms_u / best["ms"], 3)
                out["traffic_ratio"] = round(best["bytes"] / b_u, 3)
                out["fusion_efficiency"] = round((best["bytes"] / b_u) / (best["ms"] / ms_u), 3)   # Eq. 12
                out["best_plan"] = best["plan"]
                out["compulsory_tbs"] = round(best["bytes"] / (best["ms"] * 1e-3) / 1e12, 3)
            print(json.dumps(out), flush=True)
            del dev
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
