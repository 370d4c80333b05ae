"""Calibration rows for tools/round2/model_fit2.py: per (plan, autotune candidate, group) the measured
time and the model inputs printed by model_time under KF_DEBUG_MODEL.
  python tools/round2/model_fit2_data.py <bench.json> ... > profiles/round2_model_fit2_data.jsonl"""
import json, sys, re, subprocess, os
sys.path.insert(0, '/root/repo')
def comps(plan, cfg):
    code = r'''
import sys, json
sys.path.insert(0, "/root/repo")
import paper_conf_sc_wahibm14_b200 as kf, bench
wl = bench.Workload("weather", 1)
prog = kf.Program(wl.desc)
t = kf.Target(**dict(bench.cand_kw(dict(wl.tkw), json.loads(%r)), ghostwrite=0))
per, _, _ = prog.project(json.loads(%r), t)
''' % (json.dumps(cfg), json.dumps(plan))
    out = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, env=dict(os.environ, KF_DEBUG_MODEL="1"))
    res = []
    for line in out.stderr.splitlines():
        if not line.startswith('model:'): continue
        m = re.search(r"smem ([\d.]+) ms .*comp ([\d.]+) ms, ctas (\d+) warps ([\d.]+) \| bytes (\d+) threads (\d+) smemB (\d+) need (\d+) pts (\d+) thrld (\d+) depth (\d+) u (\d+) pair (\d+)", line)
        res.append(dict(smem=float(m[1]), comp=float(m[2]), bytes=int(m[5]), threads=int(m[6]), smemB=int(m[7]), need=int(m[8]), pts=int(m[9]), thrld=int(m[10]), depth=int(m[11]), u=int(m[12]), pair=int(m[13])))
    return res
for path in sys.argv[1:]:
    d = json.loads(open(path).read().strip().splitlines()[-1])
    plan = d['config']['plan_labels']
    for tr in d['config'].get('autotune_tried') or []:
        cs = comps(plan, tr['config'])
        for g, ms in enumerate(tr['group_ms']):
            if g < len(cs):
                r = dict(cs[g]); r['ms'] = ms; r['cfg'] = tr['config']; r['g'] = g; r['src'] = os.path.basename(path)
                print(json.dumps(r))
