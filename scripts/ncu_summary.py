"""Summarise an ncu --set full report: one block per profiled launch with the metrics the roofline needs."""
import csv
import subprocess
import sys

KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("sm__cycles_elapsed.avg.per_second", "sm clock"),
    ("sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed", "tensor pipe active %"),
    ("sm__mem_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed", "tensor mem (TMEM/smem) active %"),
    ("dram__bytes_read.sum", "dram read"),
    ("dram__bytes_write.sum", "dram write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram throughput %"),
    ("lts__t_bytes.sum", "L2 bytes"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "L2 throughput %"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smem LSU wavefronts"),
    ("l1tex__throughput.avg.pct_of_peak_sustained_elapsed", "L1 throughput %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("launch__registers_per_thread", "regs/thread"),
    ("launch__grid_size", "grid"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM throughput %"),
]


def main(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    h, units = rows[0], rows[1]
    for r in rows[2:]:
        print("=====", r[h.index("Kernel Name")][:110])
        for k, label in KEYS:
            if k in h:
                i = h.index(k)
                print(f"  {label:34s} {r[i]:>16s} {units[i]}")
        stalls = [(h[i], r[i]) for i in range(len(h)) if h[i].startswith("smsp__average_warp_latency_issue_stalled")
                  or h[i].startswith("smsp__pcsamp_warps_issue_stalled_")]
        top = []
        for name, v in stalls:
            try:
                top.append((float(v.replace(",", "")), name))
            except ValueError:
                pass
        for v, name in sorted(top, reverse=True)[:8]:
            print(f"  stall {name:70s} {v}")


if __name__ == "__main__":
    main(sys.argv[1])
