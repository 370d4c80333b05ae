"""One small fused run for compute-sanitizer (racecheck / synccheck / initcheck / memcheck).

  python tools/round2/sanitize_run.py tiny
  python tools/round2/sanitize_run.py weather [pairs|pairs_chunks|points]

weather: 64x48x12 fp64 weather program, HGGA plan (seed 1), every group under the knobs the bench
times (canvas pairs + pair z-queues + unpredicated canvas loads, or one point per thread), 2 steps,
checked bit for bit against the oracle afterwards (the sanitizer run must also be a correct run)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_sc_wahibm14_b200 as kf  # noqa: E402
from oracle import interp  # noqa: E402
from tests.gpu_util import compare  # noqa: E402
from workloads import data as D  # noqa: E402
from workloads import programs as P  # noqa: E402


def main():
    which = sys.argv[1] if len(sys.argv) > 1 else "tiny"
    mode = sys.argv[2] if len(sys.argv) > 2 else "pairs"
    torch.cuda.set_device(0)
    if which == "tiny":
        desc = P.tiny()
        inputs = D.uniform(desc, 1)
        plan, tgt = [0, 0, 1], kf.Target(tile=(32, 16, 0))
    else:
        desc = P.weather(n=(64, 48, 12))
        inputs = D.weather_inputs(desc, 3)
        prog0 = kf.Program(desc)
        if mode == "pairs":
            tgt = kf.Target(tile=(32, 8, 0), pblock=(2, 1), pair_zq=1, canvas_ld=1, minblocks=-1)
        elif mode == "pairs_chunks":   # z chunks of 5 planes: partial canvas iterations at chunk boundaries
            tgt = kf.Target(tile=(32, 8, 5), pblock=(2, 1), pair_zq=1, canvas_ld=1, minblocks=-1)
        else:
            tgt = kf.Target(tile=(32, 8, 0), pblock=(1, 1), canvas_ld=1, minblocks=-1)
        plan, _ = prog0.search(kf.SEARCH_HGGA, tgt, seed=1)   # legal under this launch configuration (V8)
    prog = kf.Program(desc)
    ex = kf.Exec(prog, plan, tgt)
    ex.set_graph(False)
    dev = kf.device_arrays(prog, inputs)
    sb = ex.scratch_bytes()
    scr = torch.empty(sb, dtype=torch.uint8, device="cuda") if sb else None
    ex.run(dev, scr, 2)
    torch.cuda.synchronize()
    got = kf.host_arrays(prog, dev)
    bad = compare(desc, got, interp.run(desc, inputs, 2))
    names = [ex.group_info(g).name.decode() for g in range(ex.info().n_groups)]
    print(f"[sanitize_run] {which}/{mode}: plan {plan} groups {names} parity {'OK' if not bad else bad}")
    sys.exit(1 if bad else 0)


if __name__ == "__main__":
    main()
