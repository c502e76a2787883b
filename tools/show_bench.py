"""Pretty-print bench.py JSON lines (dev helper)."""
import json
import sys

for f in sys.argv[1:]:
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:  # noqa: BLE001
        print(f, "ERR", e)
        continue
    print(f, "value %.3g %s" % (d["value"], d["unit"]), "ms %.2f" % d["ms_per_step"],
          "hier GB/s %.0f (%.1f%%)" % (d["hierarchy_GBps"], 100 * d["hierarchy_frac_of_peak"]),
          d["config"]["levels"])
    r = d["roofline"]
    print("  roofline %s %.0f GB/s frac %.3f (%.2f ms) traffic %s" % (r["kernel"], r["achieved"], r["frac"],
                                                                      r.get("ms", 0), r["traffic"]))
    for lv in d.get("levels", []):
        print("   L%d n=%d nnz=%d -> %s: %.3f ms (map %.3f, build %.3f) B=%.2f GB frac %s" % (
            lv["level"], lv["n"], lv["nnz"], lv["n_c"], lv["ms"], lv["mapping_ms"], lv["construction_ms"],
            lv["B"] / 1e9, "%.3f" % lv["frac"] if lv["frac"] else None))
    for k, v in d["phases"].items():
        print("   %-12s %8.3f ms  %7.0f GB/s  %.2f" % (k, v["ms_per_step"], v["GBps"], v["share"]))
    print("  e2e", d.get("e2e"), "\n  cpu", d.get("cpu_baseline"))
    print("  launches/step", d["gpu_launches_per_step"], "clocks", d["clocks"])
