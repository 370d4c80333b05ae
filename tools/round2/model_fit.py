"""NEXT-2 calibration data: per (plan, autotune candidate, group) the measured time from a bench
JSON's autotune_tried and the resource-aware model's components (KF_DEBUG_MODEL print of
model_time: t_mem, t_smem, t_comp).  Prints JSON lines for fitting."""
import io, json, os, re, subprocess, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))

def components(plan, cfg, workload="weather"):
    code = r'''
import sys, json
sys.path.insert(0, %r)
import paper_conf_sc_wahibm14_b200 as kf, bench
wl = bench.Workload(%r, 1)
prog = kf.Program(wl.desc)
t = kf.Target(**dict(bench.cand_kw(dict(wl.tkw), json.loads(%r)), ghostwrite=0))
per, _, _ = prog.project(json.loads(%r), t)
print("MODEL", json.dumps([g.t_model_s for g in per]))
''' % (os.getcwd(), workload, json.dumps(cfg), json.dumps(plan))
    out = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, env=dict(os.environ, KF_DEBUG_MODEL="1"))
    comps = [tuple(float(x) for x in m) for m in re.findall(r"mem ([\d.]+) ms, smem ([\d.]+) ms .* comp ([\d.]+) ms", out.stderr)]
    return comps

def main(path):
    d = json.load(open(path))
    plan = d["config"]["plan_labels"]
    for tr in d["config"]["autotune_tried"] or []:
        comps = components(plan, tr["config"])
        for g, ms in enumerate(tr["group_ms"]):
            if g < len(comps):
                print(json.dumps({"cfg": tr["config"], "g": g, "ms": ms, "mem": comps[g][0], "smem": comps[g][1], "comp": comps[g][2]}))

if __name__ == "__main__":
    main(sys.argv[1])
