"""Thin Python binding over the C ABI (include/kf.h).  Argument marshalling only:
every step of the hot path runs in libkf.so (host C++) and its sm_100a kernels.
PyTorch supplies device memory and streams."""
from __future__ import annotations

import ctypes as C
from typing import Dict, List, Optional, Sequence, Tuple

import numpy as np

from ._abi import (check, kf_access, kf_array_desc, kf_array_info, kf_box, kf_edge, kf_exec_info, kf_group_info,
                   kf_group_proj, kf_insn, kf_kernel_desc, kf_kernel_sched, kf_layout, kf_program_desc,
                   kf_program_info, kf_stmt, kf_target, kf_violation, lib)

SEARCH_BRUTE, SEARCH_GREEDY, SEARCH_AUTO, SEARCH_GREEDY_TIME, SEARCH_BRUTE_TIME, SEARCH_HGGA, SEARCH_HGGA_BYTES = range(7)


def _i32(seq) -> C.Array:
    return (C.c_int32 * len(seq))(*[int(v) for v in seq])


class Target:
    """kf_target (Table IV analogue); defaults from kf_target_b200()."""

    def __init__(self, **kw):
        t = kf_target()
        check(lib().kf_target_b200(C.byref(t)))
        for k, v in kw.items():
            if k in ("tile", "pblock"):
                arr = getattr(t, k)
                for i, x in enumerate(v):
                    arr[i] = int(x)
            else:
                setattr(t, k, v)
        self.c = t

    def __getattr__(self, k):
        if k in ("tile", "pblock"):
            return tuple(getattr(self.__dict__["c"], k))
        return getattr(self.__dict__["c"], k)


class Program:
    """Owns a kf_program handle built from a workloads.program.Program description."""

    def __init__(self, desc):
        self.desc = desc
        keep = []
        arrays = (kf_array_desc * len(desc.arrays))()
        for i, (nm, fl) in enumerate(desc.arrays):
            b = nm.encode()
            keep.append(b)
            arrays[i].name = b
            arrays[i].flags = fl
        kernels = (kf_kernel_desc * len(desc.kernels))()
        for k, kern in enumerate(desc.kernels):
            stmts = (kf_stmt * len(kern.stmts))()
            for s, st in enumerate(kern.stmts):
                ins = (kf_insn * len(st.rpn))()
                for j, x in enumerate(st.rpn):
                    ins[j].op = x.op
                    ins[j].arg = x.arg
                    for a in range(3):
                        ins[j].d[a] = x.d[a]
                    ins[j].imm = x.imm
                keep.append(ins)
                stmts[s].out_array = st.out
                stmts[s].n_insn = len(st.rpn)
                stmts[s].insn = ins
            rd = [(a, d) for a, offs in kern.reads().items() for d in offs]
            acc = (kf_access * max(1, len(rd)))()
            for j, (a, d) in enumerate(rd):
                acc[j].array = a
                for t in range(3):
                    acc[j].d[t] = d[t]
            keep += [stmts, acc]
            nb = kern.name.encode()
            keep.append(nb)
            kernels[k].name = nb
            kernels[k].n_stmt = len(kern.stmts)
            kernels[k].stmt = stmts
            kernels[k].n_reads = len(rd)
            kernels[k].reads = acc
        d = kf_program_desc()
        d.dtype = desc.dtype
        for a in range(3):
            d.n[a] = desc.n[a]
            d.ghost[a] = desc.ghost[a]
            d.bc[a] = desc.bc[a]
        d.n_arrays = len(desc.arrays)
        d.arrays = arrays
        d.n_kernels = len(desc.kernels)
        d.kernels = kernels
        d.n_params = len(desc.params)
        d.flags = desc.flags
        h = C.c_void_p()
        check(lib().kf_program_create(C.byref(d), C.byref(h)))
        self.h = h
        self.nk = len(desc.kernels)
        self.na = len(desc.arrays)

    def __del__(self):
        h = getattr(self, "h", None)
        if h:
            lib().kf_program_destroy(h)
            self.h = None

    # ---- queries
    def info(self) -> kf_program_info:
        r = kf_program_info()
        check(lib().kf_program_get_info(self.h, C.byref(r)))
        return r

    def edges(self) -> List[Tuple[int, int, int, int]]:
        n = C.c_int32()
        check(lib().kf_program_edges(self.h, None, 0, C.byref(n)))
        buf = (kf_edge * max(1, n.value))()
        check(lib().kf_program_edges(self.h, buf, n.value, C.byref(n)))
        return [(e.src, e.dst, e.kind, e.array) for e in buf[:n.value]]

    def reach(self) -> np.ndarray:
        buf = (C.c_uint8 * (self.nk * self.nk))()
        check(lib().kf_program_reach(self.h, buf))
        return np.frombuffer(buf, dtype=np.uint8).reshape(self.nk, self.nk).astype(bool)

    def array_info(self, x: int) -> kf_array_info:
        r = kf_array_info()
        check(lib().kf_program_array_info(self.h, x, C.byref(r)))
        return r

    def array_classes(self) -> List[int]:
        out = (C.c_int32 * self.na)()
        check(lib().kf_program_array_class(self.h, out))
        return list(out)

    def kinship(self, a: int, b: int, group: Sequence[int]) -> int:
        d = C.c_int32()
        check(lib().kf_program_kinship(self.h, a, b, _i32(group), len(group), C.byref(d)))
        return d.value

    def layout(self) -> kf_layout:
        r = kf_layout()
        check(lib().kf_array_layout(self.h, C.byref(r)))
        return r

    def validate(self, plan: Sequence[int], target: Optional[Target] = None) -> Tuple[int, int, int, int, int]:
        t = (target or Target()).c
        w = kf_violation()
        st = lib().kf_plan_validate(self.h, _i32(plan), C.byref(t), C.byref(w))
        if st not in (0, 3):
            check(st)
        return (w.code, w.group, w.kernel_a, w.kernel_b, w.array)

    def project(self, plan: Sequence[int], target: Optional[Target] = None):
        t = (target or Target()).c
        m = C.c_int32()
        tb = C.c_uint64()
        tt = C.c_double()
        per = (kf_group_proj * self.nk)()
        check(lib().kf_project(self.h, _i32(plan), C.byref(t), per, self.nk, C.byref(m), C.byref(tb), C.byref(tt)))
        return list(per[:m.value]), tb.value, tt.value

    def schedule(self, plan: Sequence[int], group: int, target: Optional[Target] = None):
        t = (target or Target()).c
        n = C.c_int32()
        out = (kf_kernel_sched * self.nk)()
        check(lib().kf_group_schedule(self.h, _i32(plan), C.byref(t), group, out, self.nk, C.byref(n)))
        return list(out[:n.value])

    def search(self, method=SEARCH_AUTO, target: Optional[Target] = None, seed: int = 0):
        t = (target or Target()).c
        out = (C.c_int32 * self.nk)()
        b = C.c_uint64()
        check(lib().kf_plan_search(self.h, C.byref(t), method, seed, out, C.byref(b)))
        return list(out), b.value

    def count_legal(self, target: Optional[Target] = None) -> int:
        t = (target or Target()).c
        c = C.c_uint64()
        check(lib().kf_plan_count_legal(self.h, C.byref(t), C.byref(c)))
        return c.value

    def legal_plans(self, target: Optional[Target] = None) -> List[List[int]]:
        """Every legal partition (kf_plan_enumerate; n <= 14)."""
        t = (target or Target()).c
        n = C.c_int64()
        check(lib().kf_plan_enumerate(self.h, C.byref(t), None, 0, C.byref(n)))
        buf = (C.c_int32 * max(1, n.value * self.nk))()
        check(lib().kf_plan_enumerate(self.h, C.byref(t), buf, n.value, C.byref(n)))
        return [list(buf[i * self.nk:(i + 1) * self.nk]) for i in range(n.value)]

    def jit_check(self, plan, group, target: Optional[Target] = None):
        t = (target or Target()).c
        regs, spill = C.c_int32(), C.c_int32()
        log = C.create_string_buffer(1 << 16)
        check(lib().kf_jit_check(self.h, _i32(plan), C.byref(t), group, C.byref(regs), C.byref(spill), log, 1 << 16))
        return regs.value, spill.value, log.value.decode(errors="replace")

    # ---- §8(b) one-call interface (kf_run / kf_scratch_bytes / kf_dist_init)
    def scratch_bytes(self, plan: Optional[Sequence[int]] = None) -> int:
        b = C.c_uint64()
        check(lib().kf_scratch_bytes(self.h, _i32(plan) if plan is not None else None, C.byref(b)))
        return b.value

    def run(self, plan: Sequence[int], tensors, scratch, nsteps: int, params=None, stream=None):
        """kf_run: JIT once per plan (cached in the program handle), then launch nsteps steps."""
        import torch
        if stream is None:
            stream = torch.cuda.current_stream()
        arr = (C.c_void_p * len(tensors))(*[t.data_ptr() for t in tensors])
        sp = scratch.data_ptr() if scratch is not None else 0
        sb = scratch.numel() * scratch.element_size() if scratch is not None else 0
        prm = params if params is not None else self.desc.params
        pr = (C.c_double * max(1, len(prm)))(*prm)
        check(lib().kf_run(self.h, _i32(plan), arr, C.c_void_p(sp), sb, nsteps, pr, C.c_void_p(stream.cuda_stream)))

    def dist_init(self, rank: int, world: int, px: int, py: int, nccl_id: Optional[bytes] = None):
        idb = (C.c_uint8 * 128)(*nccl_id) if nccl_id is not None else None
        check(lib().kf_dist_init(self.h, rank, world, px, py, idb))

    def dist_strips(self, axis: int):
        """Halo strips of this (local) program: [send_lo, send_hi, recv_lo, recv_hi] as
        (offset, w, h, d) in elements of the kf layout (kf_dist_strips)."""
        out = (kf_box * 4)()
        check(lib().kf_dist_strips(self.h, axis, out))
        return [(b.offset, b.w, b.h, b.d) for b in out]

    # ---- layout helpers (plumbing between the logical ghosted numpy layout and device memory)
    def to_device_layout(self, arr: np.ndarray) -> np.ndarray:
        L = self.layout()
        d = self.desc
        nz2 = d.n[2] + 2 * d.ghost[2]
        out = np.zeros(L.elems, dtype=arr.dtype)
        v = out.reshape(nz2, L.rows, L.pitch)
        gx = d.ghost[0]
        v[:, :, L.xoff - gx:L.xoff + d.n[0] + gx] = arr
        return out

    def from_device_layout(self, flat: np.ndarray) -> np.ndarray:
        L = self.layout()
        d = self.desc
        nz2 = d.n[2] + 2 * d.ghost[2]
        v = flat[:L.elems].reshape(nz2, L.rows, L.pitch)
        gx = d.ghost[0]
        return v[:, :, L.xoff - gx:L.xoff + d.n[0] + gx].copy()


class Exec:
    """kf_exec: a validated, lowered and JIT-compiled plan (one sm_100a kernel per group)."""

    def __init__(self, program: Program, plan: Sequence[int], target: Optional[Target] = None,
                 group_targets: Optional[Sequence[Target]] = None):
        self.program = program
        self.target = target or Target()
        h = C.c_void_p()
        if group_targets:
            arr = (kf_target * len(group_targets))(*[t.c for t in group_targets])
            check(lib().kf_exec_create_ex(program.h, _i32(plan), arr, len(group_targets), C.byref(h)))
        else:
            check(lib().kf_exec_create(program.h, _i32(plan), C.byref(self.target.c), C.byref(h)))
        self.h = h
        self.plan = list(plan)

    def __del__(self):
        h = getattr(self, "h", None)
        if h:
            lib().kf_exec_destroy(h)
            self.h = None

    def scratch_bytes(self) -> int:
        b = C.c_uint64()
        check(lib().kf_exec_scratch_bytes(self.h, C.byref(b)))
        return b.value

    def info(self) -> kf_exec_info:
        r = kf_exec_info()
        check(lib().kf_exec_get_info(self.h, C.byref(r)))
        return r

    def group_info(self, g: int) -> kf_group_info:
        r = kf_group_info()
        check(lib().kf_exec_group_info(self.h, g, C.byref(r)))
        return r

    def group_source(self, g: int) -> str:
        n = C.c_int64()
        check(lib().kf_exec_group_source(self.h, g, None, 0, C.byref(n)))
        buf = C.create_string_buffer(n.value + 1)
        check(lib().kf_exec_group_source(self.h, g, buf, n.value + 1, C.byref(n)))
        return buf.value.decode()

    def set_profiling(self, on: bool):
        check(lib().kf_exec_set_profiling(self.h, int(on)))

    def set_graph(self, on: bool):
        check(lib().kf_exec_set_graph(self.h, int(on)))

    def load(self):
        """kf_exec_load: load every group kernel onto the current device (NUM_REGS / LOCAL_SIZE)."""
        check(lib().kf_exec_load(self.h))

    def invalidate(self):
        """kf_exec_invalidate: array contents outside the interior changed under the same pointers."""
        check(lib().kf_exec_invalidate(self.h))

    def group_times(self):
        n = C.c_int32()
        ln = C.c_int64()
        buf = (C.c_double * 4096)()
        check(lib().kf_exec_group_times(self.h, buf, 4096, C.byref(n), C.byref(ln)))
        return list(buf[:n.value]), ln.value

    def run_ptrs(self, ptrs: Sequence[int], scratch_ptr: int, scratch_bytes: int, nsteps: int,
                 params: Optional[Sequence[float]] = None, stream: int = 0):
        arr = (C.c_void_p * len(ptrs))(*ptrs)
        prm = params if params is not None else self.program.desc.params
        pr = (C.c_double * max(1, len(prm)))(*prm)
        check(lib().kf_exec_run(self.h, arr, C.c_void_p(scratch_ptr), scratch_bytes, nsteps, pr, C.c_void_p(stream)))

    def run(self, tensors, scratch, nsteps: int, params=None, stream=None):
        """tensors: list of CUDA tensors (flat, kf layout); scratch: CUDA uint8 tensor or None."""
        import torch
        if stream is None:
            stream = torch.cuda.current_stream()
        sp = scratch.data_ptr() if scratch is not None else 0
        sb = scratch.numel() * scratch.element_size() if scratch is not None else 0
        self.run_ptrs([t.data_ptr() for t in tensors], sp, sb, nsteps, params, stream.cuda_stream)

    def run_host(self, host_ptrs: Sequence[int], nsteps: int, params=None, stream: int = 0):
        arr = (C.c_void_p * len(host_ptrs))(*host_ptrs)
        prm = params if params is not None else self.program.desc.params
        pr = (C.c_double * max(1, len(prm)))(*prm)
        h2d, d2h = C.c_uint64(), C.c_uint64()
        check(lib().kf_run_host(self.h, arr, nsteps, pr, C.c_void_p(stream), C.byref(h2d), C.byref(d2h)))
        return h2d.value, d2h.value


def flush_l2(buf, stream=None):
    import torch
    s = (stream or torch.cuda.current_stream()).cuda_stream
    check(lib().kf_flush_l2(C.c_void_p(buf.data_ptr()), buf.numel() * buf.element_size(), C.c_void_p(s)))


def device_arrays(program: Program, np_arrays: Dict[str, np.ndarray], device="cuda"):
    """Upload logical ghosted numpy arrays into kf-layout CUDA tensors (one per array)."""
    import torch
    out = []
    for nm, _ in program.desc.arrays:
        flat = program.to_device_layout(np_arrays[nm])
        out.append(torch.from_numpy(flat).to(device))
    return out


def host_arrays(program: Program, tensors) -> Dict[str, np.ndarray]:
    return {nm: program.from_device_layout(t.cpu().numpy()) for (nm, _), t in zip(program.desc.arrays, tensors)}


class Dist:
    """kf_dist: a plan run over a px x py domain decomposition (include/kf.h, row a11).

    Loopback (one process, one GPU): Dist(parts=[Exec]*px*py, px, py).
    NCCL (one process per GPU): Dist([Exec], px, py, rank, world, nccl_id)."""

    def __init__(self, parts: Sequence[Exec], px: int, py: int, rank: int = 0, world: int = 1,
                 nccl_id: Optional[bytes] = None):
        self.parts = list(parts)
        hs = (C.c_void_p * len(parts))(*[e.h for e in parts])
        idb = (C.c_uint8 * 128)(*nccl_id) if nccl_id is not None else None
        h = C.c_void_p()
        check(lib().kf_dist_create(hs, len(parts), px, py, rank, world, idb, C.byref(h)))
        self.h = h

    def __del__(self):
        h = getattr(self, "h", None)
        if h:
            lib().kf_dist_destroy(h)
            self.h = None

    def set_overlap(self, on: bool):
        """Exchange / interior-compute overlap (kf_dist_set_overlap; default on)."""
        check(lib().kf_dist_set_overlap(self.h, 1 if on else 0))

    def set_graph(self, on: bool):
        """CUDA graph of one replay period (kf_dist_set_graph; default on)."""
        check(lib().kf_dist_set_graph(self.h, 1 if on else 0))

    def run(self, part_tensors, part_scratch, nsteps: int, params=None, stream=None):
        import torch
        stream = stream or torch.cuda.current_stream()
        ptrs = [t.data_ptr() for ts in part_tensors for t in ts]
        arr = (C.c_void_p * len(ptrs))(*ptrs)
        scr = [s.data_ptr() if s is not None else 0 for s in part_scratch]
        sb = min([s.numel() * s.element_size() for s in part_scratch if s is not None] or [0])
        sarr = (C.c_void_p * len(scr))(*scr)
        prm = params if params is not None else self.parts[0].program.desc.params
        pr = (C.c_double * max(1, len(prm)))(*prm)
        check(lib().kf_dist_run(self.h, arr, sarr, sb, nsteps, pr, C.c_void_p(stream.cuda_stream)))


def dist_unique_id() -> bytes:
    buf = (C.c_uint8 * 128)()
    check(lib().kf_dist_unique_id(buf))
    return bytes(buf)


def dist_neighbors(px: int, py: int, rank: int):
    out = (C.c_int32 * 4)()
    check(lib().kf_dist_neighbors(px, py, rank, out))
    return list(out)


def split_domain(global_desc, arrays: Dict[str, np.ndarray], px: int, py: int):
    """Cut logical ghosted global arrays into px*py local ones (part-major, iy*px+ix) -- plumbing."""
    nx, ny, nz = global_desc.n
    gx, gy, gz = global_desc.ghost
    assert nx % px == 0 and ny % py == 0, "grid must divide evenly"
    lx, ly = nx // px, ny // py
    parts = []
    for iy in range(py):
        for ix in range(px):
            parts.append({nm: np.ascontiguousarray(a[:, iy * ly:iy * ly + ly + 2 * gy, ix * lx:ix * lx + lx + 2 * gx])
                          for nm, a in arrays.items()})
    return parts, global_desc.with_(n=(lx, ly, nz))


def gather_domain(global_desc, parts: Sequence[Dict[str, np.ndarray]], px: int, py: int, base: Dict[str, np.ndarray]):
    """Inverse of split_domain for the interiors (ghost cells taken from `base`)."""
    nx, ny, nz = global_desc.n
    gx, gy, gz = global_desc.ghost
    lx, ly = nx // px, ny // py
    out = {nm: a.copy() for nm, a in base.items()}
    for r, part in enumerate(parts):
        ix, iy = r % px, r // px
        for nm, a in part.items():
            out[nm][gz:gz + nz, gy + iy * ly:gy + (iy + 1) * ly, gx + ix * lx:gx + (ix + 1) * lx] = \
                a[gz:gz + nz, gy:gy + ly, gx:gx + lx]
    return out
