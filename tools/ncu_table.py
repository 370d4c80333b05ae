"""Summarise an ncu --set full report (raw page) into the table used in profiles/*.md."""
import csv, io, subprocess, sys

M = [("gpu__time_duration.sum", "dur us", "time"), ("dram__bytes_read.sum", "dram rd GB", None),
     ("dram__bytes_write.sum", "dram wr GB", None), ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram %", 1),
     ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed", "smem wf %", 1),
     ("l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum", "ld wf M", 1e-6),
     ("l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum", "st wf M", 1e-6),
     ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue %", 1),
     ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps %", 1),
     ("launch__occupancy_limit_shared_mem", "cta/sm smem", 1), ("launch__occupancy_limit_registers", "cta/sm regs", 1),
     ("launch__registers_per_thread", "regs", 1), ("launch__block_size", "threads", 1),
     ("smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio", "st barrier", 1),
     ("smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio", "st long_sb", 1),
     ("smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio", "st short_sb", 1),
     ("smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio", "st mio", 1),
     ("smsp__average_warps_issue_stalled_wait_per_issue_active.ratio", "st wait", 1),
     ("l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "bank confl M", 1e-6)]

def main(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, data = rows[0], rows[1], rows[2:]
    ix = {h: i for i, h in enumerate(hdr)}
    names = [r[ix["Kernel Name"]][:22] for r in data]
    print("| metric | " + " | ".join(names) + " |")
    print("|---" * (len(names) + 1) + "|")
    for key, lab, sc in M:
        if key not in ix:
            continue
        vals = []
        for r in data:
            v = float(r[ix[key]].replace(",", "")) if r[ix[key]] else float("nan")
            if sc == "time":   # to microseconds whatever unit ncu chose
                v *= {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3, "second": 1e6, "s": 1e6}.get(units[ix[key]], 1.0)
            elif sc is None:   # to GB
                v *= {"byte": 1e-9, "Kbyte": 1e-6, "KB": 1e-6, "Mbyte": 1e-3, "MB": 1e-3, "Gbyte": 1.0, "GB": 1.0, "Tbyte": 1e3}.get(units[ix[key]], 1e-9)
            else:
                v *= sc
            vals.append(f"{v:.3g}")
        print(f"| {lab} | " + " | ".join(vals) + " |")

if __name__ == "__main__":
    main(sys.argv[1])
