"""Summarise an ncu report into a per-launch table (dev helper; output goes to profiles/).

    python tools/ncu_summary.py gpurun_out/prof.ncu-rep [label]
"""
import csv
import io
import subprocess
import sys

METRICS = [
    ("Kernel Name", "kernel"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("launch__registers_per_thread", "regs"),
    ("gpu__time_duration.sum", "time"),
    ("dram__bytes_read.sum", "dram_rd"),
    ("dram__bytes_write.sum", "dram_wr"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram_%"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm_%"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps_active_%"),
    ("smsp__inst_executed.sum", "inst"),
    # tensor pipes: tcgen05 (hmma subpipe, UTC*MMA) and DMMA (fp64 mma.sync)
    ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", "tensor_pipe_%"),
    ("sm__pipe_tensor_subpipe_hmma_cycles_active.avg.pct_of_peak_sustained_active", "hmma_subpipe_%"),
    ("sm__pipe_tensor_subpipe_dmma_cycles_active.avg.pct_of_peak_sustained_active", "dmma_subpipe_%"),
    ("sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_active", "tc_pipe_%"),
    ("l1tex__throughput.avg.pct_of_peak_sustained_active", "l1tex_%"),
]


def main():
    rep = sys.argv[1]
    label = sys.argv[2] if len(sys.argv) > 2 else rep
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units, data = rows[0], rows[1], rows[2:]
    cols = [(hdr.index(m), name, units[hdr.index(m)]) for m, name in METRICS if m in hdr]
    print(f"# ncu --set full summary: {label}\n")
    print("| " + " | ".join(f"{n} ({u})" if u else n for _, n, u in cols) + " |")
    print("|" + "---|" * len(cols))
    for r in data:
        vals = []
        for i, n, _ in cols:
            v = r[i]
            if n == "kernel":
                v = v.split("(")[0].replace("void ", "")[-60:]
            vals.append(v)
        print("| " + " | ".join(vals) + " |")


if __name__ == "__main__":
    main()
