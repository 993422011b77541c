"""Summarise ncu outputs for profiles/ (reads gpurun_out/ artefacts here, no GPU).

usage:
  python tools/ncu_summary.py launches <launches.csv>        # per-kernel share of device time
  python tools/ncu_summary.py full <prof.ncu-rep> [name]     # key metrics of a --set full capture
"""
import collections
import csv
import io
import json
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__t_bytes.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__shared_mem_per_block_dynamic", "launch__shared_mem_per_block_static"]


def launches(path):
    rows = [r for r in csv.reader(open(path)) if len(r) > 5]
    h = rows[0]
    ix = {k: i for i, k in enumerate(h)}
    agg = collections.defaultdict(lambda: [0, 0.0])
    for r in rows[1:]:
        if r[ix["Metric Name"]] != "gpu__time_duration.sum":
            continue
        name = r[ix["Kernel Name"]].split("(")[0]
        agg[name][0] += 1
        agg[name][1] += float(r[ix["Metric Value"]].replace(",", ""))
    tot = sum(v[1] for v in agg.values())
    out = ["kernel  launches  total_us  share"]
    for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
        out.append(f"{k}  {v[0]}  {v[1] / 1e3:.1f}  {100 * v[1] / tot:.1f}%")
    return "\n".join(out)


def full(path, name=None):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = dict(zip(h, r))
        if name and name not in d.get("Kernel Name", ""):
            continue
        m = {k: d.get(k) for k in KEYS if k in d}
        m["kernel"] = d.get("Kernel Name", "").split("(")[0]
        m["units"] = {k: units[h.index(k)] for k in KEYS if k in h}
        stalls = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): float(v.replace(",", ""))
                  for k, v in d.items()
                  if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")
                  and v not in ("", "0")}
        tot = sum(stalls.values()) or 1.0
        m["stall_share"] = {k: round(v / tot, 3) for k, v in sorted(stalls.items(), key=lambda x: -x[1])[:8]}
        res.append(m)
    return json.dumps(res, indent=1)


if __name__ == "__main__":
    if sys.argv[1] == "launches":
        print(launches(sys.argv[2]))
    else:
        print(full(sys.argv[2], sys.argv[3] if len(sys.argv) > 3 else None))
