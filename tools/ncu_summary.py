"""Summarise an ncu report for profiles/: key counters + top source lines by stall samples.

    python tools/ncu_summary.py gpurun_out/p_c2_num1.ncu-rep > profiles/r01_c2_numeric.txt
"""
import csv
import io
import subprocess
import sys

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "launch__registers_per_thread", "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
    "launch__grid_size", "launch__block_size", "smsp__inst_executed.sum", "smsp__thread_inst_executed_per_inst_executed.ratio", "lts__t_sector_hit_rate.pct",
    "l1tex__t_sector_hit_rate.pct", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_atom.sum",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum",
    "l1tex__t_sectors_pipe_lsu_mem_local_op_ld.sum", "l1tex__t_sectors_pipe_lsu_mem_local_op_st.sum",
    "l1tex__t_sectors_pipe_lsu_mem_global_op_st.sum", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
    "lts__t_sectors_op_write.sum", "lts__t_sectors_op_read.sum", "lts__t_sectors_op_atom.sum", "lts__t_sectors_op_red.sum",
    "smsp__sass_inst_executed_op_local_st.sum", "smsp__sass_inst_executed_op_local_ld.sum",
]


def ncu(args):
    return subprocess.run(["ncu", "-i", *args], capture_output=True, text=True).stdout


def main(rep, launch=0):
    raw = list(csv.reader(io.StringIO(ncu([rep, "--page", "raw", "--csv"]))))
    h, units, data = raw[0], raw[1], raw[2:]
    d = data[launch]
    print(f"report: {rep}  kernel: {d[h.index('Kernel Name')]}")
    for k in KEYS:
        if k in h:
            i = h.index(k)
            print(f"  {k:70s} {d[i]:>20s} {units[i]}")
    stalls = [(float(d[i] or 0), k) for i, k in enumerate(h)
              if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("_not_issued")]
    tot = sum(v for v, _ in stalls) or 1.0
    print("stall reasons (pc sampling):", ", ".join(f"{k[33:]} {100 * v / tot:.1f}%" for v, k in sorted(stalls, reverse=True)[:8]))
    src = list(csv.reader(io.StringIO(ncu([rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                                           "--launch-skip", str(launch), "--launch-count", "1"]))))
    cur, hdr, out = None, None, []
    for r in src:
        if len(r) >= 2 and r[0] == "File Path":
            cur = r[1].split("/")[-1]
            continue
        if r and r[0] == "Line No":
            hdr = r
            continue
        if hdr and r and r[0].isdigit():
            try:
                out.append((int(r[4] or 0), int(r[7] or 0), cur, r[0], r[1][:100]))
            except ValueError:
                pass
    ts = sum(o[0] for o in out) or 1
    ti = sum(o[1] for o in out) or 1
    print(f"top source lines by stall samples (total {ts}; warp instructions {ti}):")
    for o in sorted(out, reverse=True)[:20]:
        print(f"  {100 * o[0] / ts:5.1f}% stalls {100 * o[1] / ti:5.1f}% inst  {o[2]}:{o[3]}  {o[4]}")
    print("top source lines by executed warp instructions:")
    for o in sorted(out, key=lambda x: -x[1])[:40]:
        print(f"  {100 * o[0] / ts:5.1f}% stalls {100 * o[1] / ti:5.1f}% inst  {o[2]}:{o[3]}  {o[4]}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 0)
