"""Summarise an ncu --metrics gpu__time_duration.sum launch list (CSV) per kernel
(dev helper; output goes to profiles/).

    python tools/launch_summary.py gpurun_out/launches_default.csv
"""
import collections
import csv
import sys


def main():
    rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
    h = rows[0]
    ki, mi, vi = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value")
    agg = collections.OrderedDict()
    for r in rows[1:]:
        if r[mi] != "gpu__time_duration.sum":
            continue
        k = r[ki][:90]
        n, t = agg.get(k, (0, 0.0))
        agg[k] = (n + 1, t + float(r[vi].replace(",", "")))
    tot = sum(t for _, t in agg.values())
    print("| kernel | launches | avg ns | total ms | share |")
    print("|---|---|---|---|---|")
    for k, (n, t) in agg.items():
        print(f"| `{k}` | {n} | {t / n:.0f} | {t / 1e6:.3f} | {t / tot:.1%} |")


if __name__ == "__main__":
    main()
