"""Print the key numbers of bench.py JSON lines (dev helper)."""
import json
import sys


def show(d, ind="  "):
    print(ind + "value %.1f %s ms/step %.4f launches %s" % (d["value"], d.get("unit", ""), d["ms_per_step"],
                                                        d.get("gpu_launches")))
    r = d.get("reroot")
    if r:
        print(ind + "reroot sets %s->%s theory %.3f step_speedup %.3f UP speedup %.3f" % (
            r["sets_original"], r["sets"], r["theoretical_speedup"], r["step_speedup"], r["updatePartials_speedup"]))
    u = d["updatePartials"]
    print(ind + "UP ms %.4f gflops %.1f share %.2f launches/pass %.0f" % (u["ms_per_pass"], u["gflops"],
                                                                       u["share_of_step"], u["launches_per_pass"]))
    f = d["roofline"]
    print(ind + "roof achieved %.1f GB/s frac %.3f traffic %s" % (f["achieved"], f["frac"], f.get("traffic")))


for fn in sys.argv[1:]:
    try:
        d = json.loads(open(fn).read().strip().splitlines()[-1])
    except Exception as e:
        print(fn, "ERR", e)
        continue
    print("==", fn)
    show(d)
    if "e2e" in d:
        print("  e2e %.1f clk %s cpu %s" % (d["e2e"]["value"], d.get("clocks"), (d.get("cpu_baseline") or {}).get("value")))
    if d.get("hbm_regime"):
        print("  -- hbm_regime")
        show(d["hbm_regime"], "    ")
