"""kf -- B200-native fused stencil-program executor (Wahib & Maruyama, SC'14).

The hot path lives in libkf.so (C ABI, include/kf.h): program/DAG builder, legality,
projection, plan search, NVRTC-JIT'd sm_100a group kernels and the step runtime.
This package is only the ctypes binding; it never computes anything itself.
"""
from ._abi import KfError, lib  # noqa: F401
from .api import (SEARCH_AUTO, SEARCH_BRUTE, SEARCH_BRUTE_TIME, SEARCH_GREEDY, SEARCH_GREEDY_TIME,  # noqa: F401
                  SEARCH_HGGA, SEARCH_HGGA_BYTES,
                  Exec, Program, Target,
                  Dist, device_arrays, dist_neighbors, dist_unique_id, flush_l2, gather_domain, host_arrays,
                  split_domain)
