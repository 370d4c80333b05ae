"""NEXT-2 SMEM-capacity what-if (the paper's P:485 study: "running the model with 128KB and 256KB ...
projects 1.56x and 1.65x improvements"): the plan search (HGGA on the resource-aware projection,
seeds 1-3) re-run with hypothetical shared memory per CTA, reporting the best projected step time,
its compulsory bytes and the projected speedup over the unfused plan.  Codeless (no GPU): the
projection model of DESIGN R22 with CTAs/SM scaled by the hypothetical capacity.

  python tools/round2/smem_whatif.py [weather|suite] > profiles/round2_smem_whatif.json"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import paper_conf_sc_wahibm14_b200 as kf  # noqa: E402
import bench  # noqa: E402


def main():
    wl = bench.Workload(sys.argv[1] if len(sys.argv) > 1 else "weather", 1)
    prog = kf.Program(wl.desc)
    rows = []
    for kb in (48, 100, 164, 227, 256, 512):
        t = kf.Target(**dict(wl.tkw, smem_per_block=kb * 1024 - 1024 if kb != 227 else 232448))
        best = None
        for seed in (1, 2, 3):
            plan, b = prog.search(kf.SEARCH_HGGA, t, seed=seed)
            per, tb, _ = prog.project(plan, t)
            tm = sum(g.t_model_s for g in per)
            if best is None or tm < best[0]:
                best = (tm, b, len(per), max(g.smem_bytes for g in per))
        per_u, bu, _ = prog.project(list(range(prog.nk)), t)
        tu = sum(g.t_model_s for g in per_u)
        rows.append({"smem_per_cta_kb": kb, "projected_ms": best[0] * 1e3, "bytes_per_step": best[1],
                     "groups": best[2], "largest_group_smem": best[3], "unfused_projected_ms": tu * 1e3,
                     "projected_speedup": tu / best[0]})
        print(json.dumps(rows[-1]), file=sys.stderr)
    print(json.dumps({"workload": wl.label, "method": __doc__.split("\n")[0], "rows": rows}, indent=1))


if __name__ == "__main__":
    main()
