"""Summarise an ncu --set full report: one block per profiled kernel with the metrics the roofline
discussion needs (duration, DRAM bytes / throughput, L2 hit rate, tensor-pipe utilisation, occupancy,
registers, top stall reasons).  usage: python tools/ncu_summary.py REP [REP ...]"""
import csv, subprocess, sys

WANT = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "dram_read"),
    ("dram__bytes_write.sum", "dram_write"),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "dram_%peak"),
    ("lts__t_sector_hit_rate.pct", "l2_hit_%"),
    ("lts__t_bytes.sum", "l2_bytes"),
    ("sm__pipe_tensor_op_hmma_cycles_active.avg.pct_of_peak_sustained_active", "hmma_%"),
    ("sm__inst_executed_pipe_tc.avg.pct_of_peak_sustained_active", "tc_inst_%"),
    ("sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_active", "tc_pipe_%"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm_%"),
    ("gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed", "mem_%"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "occupancy_%"),
    ("launch__registers_per_thread", "regs"),
    ("launch__grid_size", "grid"),
    ("launch__shared_mem_per_block_dynamic", "dyn_smem"),
    ("sm__cycles_elapsed.avg.per_second", "sm_clock_hz"),
]


def main():
    for rep in sys.argv[1:]:
        txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
        rows = list(csv.reader(txt.splitlines()))
        if len(rows) < 3:
            print(rep, ": no data")
            continue
        hdr, units = rows[0], rows[1]
        col = {h: i for i, h in enumerate(hdr)}
        print(f"== {rep}")
        for r in rows[2:]:
            name = r[col["Kernel Name"]][:90]
            print(f"-- {r[col['ID']]} {name}")
            for m, short in WANT:
                if m in col:
                    print(f"   {short:12s} {r[col[m]]:>16s} {units[col[m]]}")
            stalls = [(h, r[i]) for h, i in col.items()
                      if h.startswith("smsp__average_warp_latency_issue_stalled_") or
                      (h.startswith("smsp__pcsamp_warps_issue_stalled_") and not h.endswith("_not_issued"))]
            vals = []
            for h, v in stalls:
                try:
                    vals.append((float(v.replace(",", "")), h))
                except ValueError:
                    pass
            vals.sort(reverse=True)
            if vals:
                print("   stalls      " + ", ".join(f"{h.split('stalled_')[-1]}={v:g}" for v, h in vals[:6]))


if __name__ == "__main__":
    main()
