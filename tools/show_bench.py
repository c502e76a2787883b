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
    print("  roofline %s %.0f GB/s frac %.3f traffic %s" % (r["kernel"], r["achieved"], r["frac"], r["traffic"]))
    for k, v in d["phases"].items():
        print("   %-12s %8.3f ms  %7.0f GB/s  %.2f" % (k, v["ms_per_step"], v["GBps"], v["share"]))
    print("  e2e", d.get("e2e"), "\n  cpu", d.get("cpu_baseline"))
    print("  launches/step", d["gpu_launches_per_step"], "clocks", d["clocks"])
