"""Turn ncu outputs in gpurun_out/ into committed summaries under profiles/.

usage: python tools/summarize_profile.py <tag> <launches.csv> [<full.ncu-rep>]

Writes
  profiles/<tag>_launches.txt   per-kernel and per-phase device time + DRAM bytes
                                (ncu --metrics gpu__time_duration.sum,dram__bytes_*,
                                cold-cache serialised launches: compare shares)
  profiles/<tag>_launches.csv   the raw launch list
  profiles/<tag>_full.txt       key --set full metrics + warp-stall breakdown
  profiles/ncu_traffic.json     DRAM bytes per level of mapping / construction, stamped
                                with the CUDA sources' hash (read by bench.py)
"""
import collections
import csv
import json
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PROF = os.path.join(ROOT, "profiles")

# kernels of the mapping (a1-a5); every other libhec kernel belongs to the construction
MAPPING = ("k_span_coords", "k_heavy", "k_fill_identity", "k_tile_coords", "k_round_init", "k_rounds",
           "RootFlagIn", "k_assign", "k_jump", "k_hkey_to_H")
# first launch of each level's mapping (k_hkey_to_H: keys fused into the previous placement;
# k_heavy_rows: small graphs)
LEVEL_START = ("k_span_coords", "k_tile_coords", "k_fill_identity", "k_hkey_to_H", "k_heavy_rows")


def part_of(name):
    return "mapping" if any(k in name for k in MAPPING) else "construction"


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr, per = None, collections.OrderedDict()
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            key = (d["ID"], d["Kernel Name"].split("(")[0].replace("void ", ""))
            per.setdefault(key, {})[d["Metric Name"]] = float(d["Metric Value"].replace(",", ""))
    return per


def main():
    tag, lc = sys.argv[1], sys.argv[2]
    os.makedirs(PROF, exist_ok=True)
    per = launches(lc)
    shutil.copy(lc, os.path.join(PROF, f"{tag}_launches.csv"))
    tot = sum(v.get("gpu__time_duration.sum", 0) for v in per.values())
    kern = collections.OrderedDict()
    for (i, k), v in per.items():
        t = v.get("gpu__time_duration.sum", 0)
        b = v.get("dram__bytes_read.sum", 0) + v.get("dram__bytes_write.sum", 0)
        for agg, key in ((kern, k),):
            a = agg.setdefault(key, [0, 0.0, 0.0])
            a[0] += 1
            a[1] += t
            a[2] += b
    lines = [f"# {tag}: ncu launch list (gpu__time_duration.sum, dram__bytes_read/write.sum), "
             f"{len(per)} launches, {tot / 1e6:.3f} ms total (cold-cache, serialised)", "", "## per kernel"]
    for k, (n, t, b) in sorted(kern.items(), key=lambda kv: -kv[1][1]):
        lines.append(f"{k[:58]:58s} n={n:4d} {t / 1e6:9.3f} ms {100 * t / tot:5.1f}%  DRAM {b / 1e9:8.3f} GB "
                     f"{b / max(t, 1):7.1f} GB/s")
    # per level (a level starts at its mapping's first launch): mapping / construction
    levels = []
    for (i, k), v in per.items():
        if any(k.startswith(x) for x in LEVEL_START) or not levels:
            levels.append({"mapping_ms": 0.0, "mapping_dram": 0.0, "construction_ms": 0.0,
                           "construction_dram": 0.0, "launches": 0})
        t = v.get("gpu__time_duration.sum", 0)
        b = v.get("dram__bytes_read.sum", 0) + v.get("dram__bytes_write.sum", 0)
        pt = part_of(k)
        levels[-1][pt + "_ms"] += t / 1e6
        levels[-1][pt + "_dram"] += b
        levels[-1]["launches"] += 1
    lines += ["", "## per level (ncu, cold-cache)"]
    for l, lv in enumerate(levels):
        lines.append(f"L{l}: mapping {lv['mapping_ms']:8.3f} ms DRAM {lv['mapping_dram'] / 1e9:7.3f} GB | "
                     f"construction {lv['construction_ms']:8.3f} ms DRAM {lv['construction_dram'] / 1e9:7.3f} GB "
                     f"({lv['launches']} launches)")
    open(os.path.join(PROF, f"{tag}_launches.txt"), "w").write("\n".join(lines) + "\n")
    # per workload (tag r2_c4_... -> "C4"): bench.py reads the entry of its own config
    cfg = next(("C" + p[1:] for p in tag.split("_") if p[:1] == "c" and p[1:].isdigit()), tag)
    tp = os.path.join(PROF, "ncu_traffic.json")
    allt = json.load(open(tp)) if os.path.exists(tp) else {}
    allt = {k: v for k, v in allt.items() if isinstance(v, dict) and "levels" in v}
    sys.path.insert(0, ROOT)
    from bench import source_stamp
    allt[cfg] = {"tag": tag, "source": f"profiles/{tag}_launches.csv", "source_stamp": source_stamp(),
                 "unit": "DRAM bytes (read + write) per hierarchy, ncu cold-cache", "levels": levels}
    json.dump(allt, open(tp, "w"), indent=1)
    print("\n".join(lines))
    if len(sys.argv) > 3:
        rep = sys.argv[3]
        raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
        r = list(csv.reader(raw.splitlines()))
        h, units, rows = r[0], r[1], r[2:]
        want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
                "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
                "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
                "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
                "smsp__inst_executed.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
                "lts__t_sector_hit_rate.pct"]
        out = [f"# {tag}: ncu --set full summary ({os.path.basename(rep)})"]
        for row in rows:
            name = row[h.index("Kernel Name")].split("(")[0]
            vals = {k: f"{row[h.index(k)]} {units[h.index(k)]}".strip() for k in want if k in h}
            st = []
            for i, k in enumerate(h):
                if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued"):
                    try:
                        st.append((float(row[i].replace(",", "")), k.replace("smsp__pcsamp_warps_issue_stalled_", "")))
                    except ValueError:
                        pass
            st.sort(reverse=True)
            s = sum(v for v, _ in st) or 1
            out.append(f"\n{name}  (launch {row[h.index('ID')]})")
            out += [f"  {k}: {v}" for k, v in vals.items()]
            out.append("  stalls: " + ", ".join(f"{k}={100 * v / s:.0f}%" for v, k in st[:8]))
        open(os.path.join(PROF, f"{tag}_full.txt"), "w").write("\n".join(out) + "\n")


if __name__ == "__main__":
    main()
