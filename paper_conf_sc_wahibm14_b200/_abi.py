"""ctypes mirror of include/kf.h (argument marshalling only)."""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libkf.so")

KF_OK = 0
STATUS = {0: "KF_OK", 1: "KF_E_ARG", 2: "KF_E_PROGRAM", 3: "KF_E_ILLEGAL_PLAN", 4: "KF_E_RESOURCE",
          5: "KF_E_CUDA", 6: "KF_E_NVRTC", 7: "KF_E_NCCL", 8: "KF_E_OOM", 9: "KF_E_UNSUPPORTED"}


class kf_insn(C.Structure):
    _fields_ = [("op", C.c_int32), ("arg", C.c_int32), ("d", C.c_int8 * 3), ("pad0", C.c_int8),
                ("pad1", C.c_int32), ("imm", C.c_double)]


class kf_stmt(C.Structure):
    _fields_ = [("out_array", C.c_int32), ("n_insn", C.c_int32), ("insn", C.POINTER(kf_insn))]


class kf_access(C.Structure):
    _fields_ = [("array", C.c_int32), ("d", C.c_int8 * 3), ("pad", C.c_int8)]


class kf_kernel_desc(C.Structure):
    _fields_ = [("name", C.c_char_p), ("n_stmt", C.c_int32), ("stmt", C.POINTER(kf_stmt)),
                ("n_reads", C.c_int32), ("reads", C.POINTER(kf_access))]


class kf_array_desc(C.Structure):
    _fields_ = [("name", C.c_char_p), ("flags", C.c_uint32)]


class kf_program_desc(C.Structure):
    _fields_ = [("dtype", C.c_int32), ("pad", C.c_int32), ("n", C.c_int64 * 3), ("ghost", C.c_int32 * 3),
                ("bc", C.c_int32 * 3), ("n_arrays", C.c_int32), ("arrays", C.POINTER(kf_array_desc)),
                ("n_kernels", C.c_int32), ("kernels", C.POINTER(kf_kernel_desc)), ("n_params", C.c_int32),
                ("flags", C.c_uint32)]


class kf_program_info(C.Structure):
    _fields_ = [("n_kernels", C.c_int32), ("n_arrays", C.c_int32), ("n_edges", C.c_int32), ("es", C.c_int32),
                ("npts", C.c_int64), ("n_relaxed", C.c_int32), ("pad", C.c_int32)]


class kf_edge(C.Structure):
    _fields_ = [("src", C.c_int32), ("dst", C.c_int32), ("kind", C.c_int32), ("array", C.c_int32)]


class kf_array_info(C.Structure):
    _fields_ = [("cls", C.c_int32), ("n_writers", C.c_int32), ("n_readers", C.c_int32), ("relaxed", C.c_int32),
                ("step_live", C.c_int32), ("upward_exposed", C.c_int32)]


class kf_layout(C.Structure):
    _fields_ = [("pitch", C.c_int64), ("rows", C.c_int64), ("plane", C.c_int64), ("origin", C.c_int64),
                ("elems", C.c_int64), ("xoff", C.c_int32), ("pad", C.c_int32)]


class kf_target(C.Structure):
    _fields_ = [("hbm_bytes_per_s", C.c_double), ("smem_per_block", C.c_int32), ("regs_per_thread_max", C.c_int32),
                ("n_sm", C.c_int32), ("tile", C.c_int32 * 3), ("stages", C.c_int32), ("threads", C.c_int32),
                ("max_halo", C.c_int32), ("internal_axes", C.c_int32), ("zunroll", C.c_int32),
                ("pblock", C.c_int32 * 2), ("ringunroll", C.c_int32), ("ghostwrite", C.c_int32),
                ("minblocks", C.c_int32), ("skew", C.c_int32), ("canvas_ld", C.c_int32), ("pair_zq", C.c_int32),
                ("inline_xy", C.c_int32)]


class kf_violation(C.Structure):
    _fields_ = [("code", C.c_int32), ("group", C.c_int32), ("kernel_a", C.c_int32), ("kernel_b", C.c_int32),
                ("array", C.c_int32)]


class kf_group_proj(C.Structure):
    _fields_ = [("bytes_read", C.c_uint64), ("bytes_written", C.c_uint64), ("halo_bytes_est", C.c_uint64),
                ("smem_bytes", C.c_uint32), ("regs_est", C.c_uint32), ("n_kernels", C.c_int32),
                ("unprofitable", C.c_int32), ("t_s", C.c_double), ("t_model_s", C.c_double)]


class kf_kernel_sched(C.Structure):
    _fields_ = [("kernel", C.c_int32), ("alive", C.c_int32), ("delay", C.c_int32), ("pad", C.c_int32),
                ("elo", C.c_int32 * 3), ("ehi", C.c_int32 * 3)]


class kf_exec_info(C.Structure):
    _fields_ = [("n_groups", C.c_int32), ("launches_per_step", C.c_int32), ("fills_per_step", C.c_int32),
                ("period", C.c_int32), ("compulsory_bytes_per_step", C.c_uint64)]


class kf_group_info(C.Structure):
    _fields_ = [("group", C.c_int32), ("grid", C.c_int32), ("threads", C.c_int32), ("smem_bytes", C.c_int32),
                ("regs", C.c_int32), ("local_bytes", C.c_int32), ("n_kernels", C.c_int32), ("max_threads", C.c_int32),
                ("bytes_per_launch", C.c_uint64), ("onchip_bytes_per_launch", C.c_uint64), ("name", C.c_char * 64)]


class kf_box(C.Structure):
    _fields_ = [("offset", C.c_int64), ("w", C.c_int32), ("h", C.c_int32), ("d", C.c_int32), ("pad", C.c_int32)]


class kf_paper_meta(C.Structure):
    _fields_ = [(n, C.c_int32) for n in ("t_b", "blocks_smx", "thr", "blocks", "hal", "halo", "shared_arrays", "smx",
                                         "r_t", "r_max", "r_smx", "r_adr", "sh_smx", "b_conf", "elem_bytes", "pad")] + \
               [(n, C.c_double) for n in ("gmem_bw_gbs", "regfac", "max_thread_load", "fl_unfused_sum", "flop_halo_sum")]


class kf_paper_proj(C.Structure):
    _fields_ = [(n, C.c_int32) for n in ("h_th", "eq2_ok", "eq3_ok", "eq6_ok", "eq7_ok", "pad")] + \
               [(n, C.c_double) for n in ("b_sh", "b_eff", "p_membound_gflops", "t_pro_s")]


P = C.c_void_p
I32P = C.POINTER(C.c_int32)
U64P = C.POINTER(C.c_uint64)

# name -> (restype, argtypes); every symbol declared in include/kf.h
SIGNATURES = {
    "kf_last_error": (C.c_char_p, []),
    "kf_version": (C.c_char_p, []),
    "kf_program_create": (C.c_int, [C.POINTER(kf_program_desc), C.POINTER(P)]),
    "kf_program_destroy": (None, [P]),
    "kf_program_get_info": (C.c_int, [P, C.POINTER(kf_program_info)]),
    "kf_program_edges": (C.c_int, [P, C.POINTER(kf_edge), C.c_int32, I32P]),
    "kf_program_reach": (C.c_int, [P, C.POINTER(C.c_uint8)]),
    "kf_program_array_info": (C.c_int, [P, C.c_int32, C.POINTER(kf_array_info)]),
    "kf_program_array_class": (C.c_int, [P, I32P]),
    "kf_program_kinship": (C.c_int, [P, C.c_int32, C.c_int32, I32P, C.c_int32, I32P]),
    "kf_array_layout": (C.c_int, [P, C.POINTER(kf_layout)]),
    "kf_target_b200": (C.c_int, [C.POINTER(kf_target)]),
    "kf_plan_validate": (C.c_int, [P, I32P, C.POINTER(kf_target), C.POINTER(kf_violation)]),
    "kf_plan_canonical": (C.c_int, [I32P, C.c_int32, I32P, I32P]),
    "kf_project": (C.c_int, [P, I32P, C.POINTER(kf_target), C.POINTER(kf_group_proj), C.c_int32, I32P, U64P,
                             C.POINTER(C.c_double)]),
    "kf_group_schedule": (C.c_int, [P, I32P, C.POINTER(kf_target), C.c_int32, C.POINTER(kf_kernel_sched),
                                    C.c_int32, I32P]),
    "kf_plan_search": (C.c_int, [P, C.POINTER(kf_target), C.c_int32, C.c_uint64, I32P, U64P]),
    "kf_plan_count_legal": (C.c_int, [P, C.POINTER(kf_target), U64P]),
    "kf_plan_enumerate": (C.c_int, [P, C.POINTER(kf_target), I32P, C.c_int64, C.POINTER(C.c_int64)]),
    "kf_exec_create": (C.c_int, [P, I32P, C.POINTER(kf_target), C.POINTER(P)]),
    "kf_exec_create_ex": (C.c_int, [P, I32P, C.POINTER(kf_target), C.c_int32, C.POINTER(P)]),
    "kf_exec_destroy": (None, [P]),
    "kf_exec_scratch_bytes": (C.c_int, [P, U64P]),
    "kf_exec_run": (C.c_int, [P, C.POINTER(P), P, C.c_uint64, C.c_int64, C.POINTER(C.c_double), P]),
    "kf_run_host": (C.c_int, [P, C.POINTER(P), C.c_int64, C.POINTER(C.c_double), P, U64P, U64P]),
    "kf_exec_get_info": (C.c_int, [P, C.POINTER(kf_exec_info)]),
    "kf_exec_group_info": (C.c_int, [P, C.c_int32, C.POINTER(kf_group_info)]),
    "kf_exec_group_source": (C.c_int, [P, C.c_int32, C.c_char_p, C.c_int64, C.POINTER(C.c_int64)]),
    "kf_exec_set_profiling": (C.c_int, [P, C.c_int32]),
    "kf_exec_group_times": (C.c_int, [P, C.POINTER(C.c_double), C.c_int32, I32P, C.POINTER(C.c_int64)]),
    "kf_exec_set_graph": (C.c_int, [P, C.c_int32]),
    "kf_exec_invalidate": (C.c_int, [P]),
    "kf_exec_load": (C.c_int, [P]),
    "kf_flush_l2": (C.c_int, [P, C.c_uint64, P]),
    "kf_paper_projection": (C.c_int, [C.POINTER(kf_paper_meta), C.POINTER(kf_paper_proj)]),
    "kf_dist_unique_id": (C.c_int, [C.POINTER(C.c_uint8)]),
    "kf_dist_neighbors": (C.c_int, [C.c_int32, C.c_int32, C.c_int32, I32P]),
    "kf_dist_create": (C.c_int, [C.POINTER(P), C.c_int32, C.c_int32, C.c_int32, C.c_int32, C.c_int32,
                                 C.POINTER(C.c_uint8), C.POINTER(P)]),
    "kf_dist_run": (C.c_int, [P, C.POINTER(P), C.POINTER(P), C.c_uint64, C.c_int64, C.POINTER(C.c_double), P]),
    "kf_dist_set_overlap": (C.c_int, [P, C.c_int32]),
    "kf_dist_destroy": (None, [P]),
    "kf_dist_set_graph": (C.c_int, [P, C.c_int32]),
    "kf_dist_strips": (C.c_int, [P, C.c_int32, C.POINTER(kf_box)]),
    "kf_dist_init": (C.c_int, [P, C.c_int32, C.c_int32, C.c_int32, C.c_int32, C.POINTER(C.c_uint8)]),
    "kf_scratch_bytes": (C.c_int, [P, I32P, U64P]),
    "kf_run": (C.c_int, [P, I32P, C.POINTER(P), P, C.c_uint64, C.c_int64, C.POINTER(C.c_double), P]),
    "kf_jit_check": (C.c_int, [P, I32P, C.POINTER(kf_target), C.c_int32, I32P, I32P, C.c_char_p, C.c_int64]),
}

_lib = None


def lib():
    """Load libkf.so (fails loudly: there is no fallback path)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is missing: run __graft_entry__.build() (no CPU fallback exists)")
        L = C.CDLL(LIB_PATH)
        for name, (res, args) in SIGNATURES.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


class KfError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


def check(st):
    if st != KF_OK:
        raise KfError(st, lib().kf_last_error().decode(errors="replace"))
