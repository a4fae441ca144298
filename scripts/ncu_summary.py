"""Summarise an ncu --set full report (per kernel launch): time, DRAM bytes and
throughput, occupancy, registers, top stall reasons.  Usage:
python scripts/ncu_summary.py report.ncu-rep"""
import csv
import subprocess
import sys

WANT = ["Kernel Name", "Grid Size", "Block Size", "gpu__time_duration.sum", "dram__bytes_read.sum",
        "dram__bytes_write.sum", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "l1tex__t_sector_hit_rate.pct",
        "lts__t_sector_hit_rate.pct", "sm__pipe_tensor_op_hmma_cycles_active.avg.pct_of_peak_sustained_active",
        "smsp__inst_executed.sum", "local_load", "local_store"]


def main(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr, units = rows[0], rows[1]
    stall_cols = [i for i, h in enumerate(hdr) if h.startswith("smsp__average_warps_issue_stalled_") and
                  h.endswith("_per_issue_active.ratio")]
    for r in rows[2:]:
        print("----")
        for w in WANT:
            for i, h in enumerate(hdr):
                if h == w or (w in ("local_load", "local_store") and h.startswith(
                        "l1tex__t_sectors_pipe_lsu_mem_local_op_" + ("ld" if w == "local_load" else "st")) and h.endswith(".sum")):
                    print(f"  {h:70s} {r[i]} {units[i]}")
        st = sorted(((float(r[i].replace(',', '')) if r[i] else 0.0, hdr[i]) for i in stall_cols), reverse=True)[:6]
        for v, h in st:
            print(f"  stall {h:64s} {v:.2f}")


if __name__ == "__main__":
    main(sys.argv[1])
