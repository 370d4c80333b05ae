"""ORACLE -- test infrastructure only.

A plain, slow, obviously-correct CPU implementation of what the fused-stencil
hot path computes, written from the paper and the readings listed in
DESIGN.md.  Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s
cpu_baseline / `--impl reference` legs may import it.  It shares no code with
the CUDA path (`paper_conf_sc_wahibm14_b200/`); both read the same program
descriptions and seeded inputs from `workloads/`.

Modules
  interp    O-1  unfused program semantics (the result the method must reproduce)
  graph     O-2/3/4  versions, precedence DAG, array classes, sharing/kinship, liveness
  legality  O-5/6/9  extended regions by point sets, V1..V8, compulsory bytes, projection
  tilesim   O-7  executes a fused group tile by tile (semantic pin for V5 and a3)
  enum      O-8  brute-force enumeration of partitions (restricted growth strings)

Parity status: every function is pinned except
the resource model of V7/V8, which is a *definition* (a contract the CUDA
kernel must stay inside), pinned only by a hand-worked example.
"""
