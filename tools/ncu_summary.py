"""Key metrics of every kernel in an ncu report: python tools/ncu_summary.py rep.ncu-rep"""
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
        "launch__registers_per_thread", "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__grid_size",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum"]
STALL = "smsp__average_warps_issue_stalled_"


def rows(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    hdr, units = r[0], r[1]
    return hdr, units, r[2:]


if __name__ == "__main__":
    hdr, units, data = rows(sys.argv[1])
    for d in data:
        name = d[hdr.index("Kernel Name")][:90]
        print("==", name)
        for k in KEYS:
            if k in hdr:
                print(f"   {k:70s} {d[hdr.index(k)]} {units[hdr.index(k)]}")
        st = [(h[len(STALL):].replace("_per_issue_active.ratio", ""), float(d[i] or 0)) for i, h in enumerate(hdr)
              if h.startswith(STALL) and h.endswith("per_issue_active.ratio")]
        st.sort(key=lambda x: -x[1])
        print("   stalls/issue:", ", ".join(f"{a}={b:.2f}" for a, b in st[:7]))
