"""Turn ncu outputs in gpurun_out/ into committed summaries under profiles/.

usage: python tools/summarize_profile.py <tag> <launches.csv> [<full.ncu-rep>]

Writes
  profiles/<tag>_launches.txt   per-kernel and per-phase device time + DRAM bytes
                                (ncu --metrics gpu__time_duration.sum,dram__bytes_*,
                                cold-cache serialised launches: compare shares)
  profiles/<tag>_launches.csv   the raw launch list
  profiles/<tag>_full.txt       key --set full metrics + warp-stall breakdown
  profiles/ncu_traffic.json     DRAM bytes per step per bench phase (read by bench.py)
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

# libhec kernel -> bench.py phase (hec_ctx_profile names)
PHASE = {
    "k_tile_coords": "heavy", "k_heavy": "heavy", "k_heavy_fixup": "heavy", "k_fill_identity": "heavy",
    "k_round_init": "rounds", "k_rounds": "rounds",
    "RootFlagIn": "relabel", "k_assign": "relabel",
    "k_member_count": "bucket", "k_member_fill": "bucket", "k_big_rows": "bucket", "CountIn": "bucket",
    "DegIn": "bucket", "RowWeightIn": "bucket", "BlockCountIn": "bucket",
    "UnitsIn": "rows_skew", "BucketsIn": "rows_skew", "k_part_count": "rows_skew", "k_part_write": "rows_skew",
    "k_fb_jobs": "rows_skew", "k_bucket_fallback": "rows_skew", "k_dense_accum": "rows_skew",
    "k_block_desc": "rows", "k_block_ends": "rows", "k_rows": "rows", "BlkCntIn": "rows",
    "k_pieces": "rows", "k_tiers": "rows", "k_wide_list": "rows", "k_expand": "expand",
    "k_bucket_blocks": "rows_skew",
    "k_place": "place", "k_hrank": "rows", "k_rbm": "rows", "k_span_coords": "heavy",
    "k_row_bins": "rows_skew", "k_part_warp": "rows_skew", "k_seg_fill": "rows_skew", "RowUIn": "rows_skew",
}


def phase_of(name):
    for k, v in PHASE.items():
        if k in name:
            return v
    return "other"


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
    kern, ph = collections.OrderedDict(), collections.OrderedDict()
    for (i, k), v in per.items():
        t = v.get("gpu__time_duration.sum", 0)
        b = v.get("dram__bytes_read.sum", 0) + v.get("dram__bytes_write.sum", 0)
        for agg, key in ((kern, k), (ph, phase_of(k))):
            a = agg.setdefault(key, [0, 0.0, 0.0])
            a[0] += 1
            a[1] += t
            a[2] += b
    lines = [f"# {tag}: ncu launch list (gpu__time_duration.sum, dram__bytes_read/write.sum), "
             f"{len(per)} launches, {tot / 1e6:.3f} ms total (cold-cache, serialised)", "", "## per kernel"]
    for k, (n, t, b) in sorted(kern.items(), key=lambda kv: -kv[1][1]):
        lines.append(f"{k[:58]:58s} n={n:4d} {t / 1e6:9.3f} ms {100 * t / tot:5.1f}%  DRAM {b / 1e9:8.3f} GB "
                     f"{b / max(t, 1):7.1f} GB/s")
    lines += ["", "## per bench phase"]
    traffic = {}
    for k, (n, t, b) in sorted(ph.items(), key=lambda kv: -kv[1][1]):
        lines.append(f"{k:12s} {t / 1e6:9.3f} ms {100 * t / tot:5.1f}%  DRAM {b / 1e9:8.3f} GB")
        traffic[k] = b
    open(os.path.join(PROF, f"{tag}_launches.txt"), "w").write("\n".join(lines) + "\n")
    # per workload (tag r1_c4_... -> "C4"): bench.py reads the entry of its own config
    cfg = next(("C" + p[1:] for p in tag.split("_") if p[:1] == "c" and p[1:].isdigit()), tag)
    tp = os.path.join(PROF, "ncu_traffic.json")
    allt = json.load(open(tp)) if os.path.exists(tp) else {}
    if "tag" in allt:  # old single-workload layout
        allt = {}
    allt[cfg] = {"tag": tag, "source": f"profiles/{tag}_launches.csv", "unit": "bytes per step", **traffic}
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
