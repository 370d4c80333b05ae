"""NEXT-2: the paper's codeless upper-bound projection, Eq. 2-10, written out
as printed (test infrastructure).  Readings: R11 (Hal in points), R12 (Eq. 10 halo term per
block and thread), R14 (the "8" of Eq. 9 is the element size in bytes)."""
import math


def project(t_b, blocks_smx, thr, blocks, hal, halo, shared_arrays, smx, gmem_bw_gbs, elem_bytes=8,
            fl_unfused_sum=0.0, flop_halo_sum=0.0):
    c = 1 if halo else 0
    h_th = math.ceil(hal / thr)
    b_sh = t_b * blocks_smx / ((1 + c * h_th) * shared_arrays)      # Eq. 8
    b_eff = b_sh * smx / (thr * blocks)
    p_mem = b_eff * gmem_bw_gbs / elem_bytes                        # Eq. 9
    flops = fl_unfused_sum + flop_halo_sum * hal / (blocks * thr)   # Eq. 10 numerator
    t_pro = flops * 1e-9 / p_mem
    return dict(h_th=h_th, b_sh=b_sh, b_eff=b_eff, p_membound_gflops=p_mem, t_pro_s=t_pro)
