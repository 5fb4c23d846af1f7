#!/usr/bin/env python
"""Print the key counters of an ncu --set full report (pipe utilisation, L1
wavefronts, DRAM bytes, issue, stalls) as `name value` lines."""
import csv
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "sm__cycles_elapsed.avg", "launch__registers_per_thread",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__inst_executed.avg.per_cycle_active",
        "smsp__inst_executed.sum", "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
        "l1tex__lsu_writeback_active.avg.pct_of_peak_sustained_elapsed", "l1tex__throughput.avg.pct_of_peak_sustained_active",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "dram__bytes.sum.per_second",
        # local memory (register spills): bytes the LSU moved, and L2 sectors of the local aperture
        "sass__inst_executed_local_loads", "sass__inst_executed_local_stores",
        "l1tex__t_sectors_pipe_lsu_mem_local_op_ld.sum", "l1tex__t_sectors_pipe_lsu_mem_local_op_st.sum",
        "l1tex__t_sectors_pipe_lsu_mem_local_op_st_lookup_miss.sum",
        "l1tex__t_output_wavefronts_pipe_lsu_mem_local_op_ld.sum", "l1tex__t_output_wavefronts_pipe_lsu_mem_local_op_st.sum"]


def main(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    h, u, v = rows[0], rows[1], rows[2]
    col = {n: i for i, n in enumerate(h)}
    for k in KEYS:
        if k in col:
            print(f"{k} {v[col[k]]} {u[col[k]]}")
    stalls = [(float(v[i]), n) for n, i in col.items()
              if n.startswith("smsp__average_warp_latency_issue_stalled") and n.endswith(".ratio") and v[i]]
    stalls += [(float(v[i]), n) for n, i in col.items()
               if n.startswith("smsp__average_warps_issue_stalled_") and n.endswith("_per_issue_active.ratio") and v[i]]
    for val, n in sorted(stalls, reverse=True)[:8]:
        print(f"{n} {val}")
    opcode_mix(path)


def opcode_mix(path, top=14):
    """Executed instructions by SASS opcode (the source page's per-instruction counters, captured
    with --import-source): `opmix OPCODE share_of_executed stall_sample_share` lines."""
    import collections
    out = subprocess.run(["ncu", "-i", path, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr = next((r for r in rows if "Instructions Executed" in r), None)
    if not hdr:
        return
    i_src, i_ex = hdr.index("Source"), hdr.index("Instructions Executed")
    i_st = hdr.index("Warp Stall Sampling (All Samples)") if "Warp Stall Sampling (All Samples)" in hdr else None
    ex, st = collections.Counter(), collections.Counter()
    for r in rows[rows.index(hdr) + 1:]:
        if len(r) <= i_ex or not r[i_ex].isdigit():
            continue
        toks = r[i_src].split()
        if not toks:
            continue
        op = (toks[1] if toks[0].startswith("@") and len(toks) > 1 else toks[0]).split(".")[0]
        ex[op] += int(r[i_ex])
        if i_st is not None and r[i_st].isdigit():
            st[op] += int(r[i_st])
    te, ts = sum(ex.values()) or 1, sum(st.values()) or 1
    for op, n in ex.most_common(top):
        print(f"opmix {op} {100.0 * n / te:.1f}% {100.0 * st[op] / ts:.1f}%")


if __name__ == "__main__":
    main(sys.argv[1])
