"""Key metrics of an ncu --set full report (ncu -i X --page raw --csv): duration, issue and pipe
utilisation, shared-memory wavefronts, DRAM bytes, occupancy, registers — one block per kernel."""
import csv
import io
import subprocess
import sys

KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("sm__inst_issued.avg.pct_of_peak_sustained_active", "issue % active"),
    ("sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", "alu pipe %"),
    ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "fma pipe %"),
    ("sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active", "xu pipe %"),
    ("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "lsu pipe %"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smem wavefronts"),
    ("l1tex__throughput.avg.pct_of_peak_sustained_active", "l1tex %"),
    ("dram__bytes_read.sum", "dram read"),
    ("dram__bytes_write.sum", "dram write"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("launch__registers_per_thread", "registers"),
    ("launch__grid_size", "grid"),
    ("sm__cycles_active.avg", "sm cycles active avg"),
    ("sm__cycles_active.max", "sm cycles active max"),
    ("smsp__average_warp_latency_issue_stalled_mio_throttle", "stall mio_throttle"),
    ("smsp__average_warp_latency_issue_stalled_short_scoreboard", "stall short_scoreboard"),
    ("smsp__average_warp_latency_issue_stalled_wait", "stall wait"),
    ("smsp__inst_executed.sum", "warp instructions"),
]


def main(rep):
    txt = subprocess.check_output(["ncu", "-i", rep, "--page", "raw", "--csv"], text=True)
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units = rows[0], rows[1]
    for r in rows[2:]:
        print(r[hdr.index("Kernel Name")][:100])
        for k, lab in KEYS:
            if k in hdr:
                j = hdr.index(k)
                print(f"  {lab:22s} {r[j]} {units[j]}")


if __name__ == "__main__":
    main(sys.argv[1])
