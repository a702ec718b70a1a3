"""Per-launch DRAM traffic of the updatePartials kernel from ncu --set full
captures (dev helper): mean of dram__bytes_read.sum + dram__bytes_write.sum over
the captured launches (one full rerooted pass each), written to
profiles/ncu_traffic.json for bench.py's roofline.traffic.

    python tools/ncu_traffic.py [--out PATH] c1_fp32=gpurun_out/prof_c1.ncu-rep c2_fp32=... c3_fp32=...
"""
import csv
import io
import json
import subprocess
import sys


def per_launch(rep):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, units, data = rows[0], rows[1], rows[2:]
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    rd, wr = h.index("dram__bytes_read.sum"), h.index("dram__bytes_write.sum")
    tot = [float(r[rd]) * scale[units[rd]] + float(r[wr]) * scale[units[wr]] for r in data]
    return sum(tot) / len(tot), len(tot)


def main():
    out = {"_note": ("dram__bytes_read.sum + dram__bytes_write.sum per updatePartials launch, averaged "
                     "over every launch of one rerooted pass captured with ncu --set full "
                     "(tools/gpu_round.sh; ncu flushes caches between kernel replays, so L2-resident "
                     "children of the launch-bound configs read as DRAM traffic). Summaries: "
                     "profiles/r01_ncu_full_*.md")}
    args = sys.argv[1:]
    path = "profiles/ncu_traffic.json"
    if args and args[0] == "--out":
        path, args = args[1], args[2:]
    for arg in args:
        key, rep = arg.split("=", 1)
        v, n = per_launch(rep)
        out[key] = round(v)
        out[key + "_launches"] = n
    json.dump(out, open(path, "w"), indent=1)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
