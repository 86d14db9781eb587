"""Turn gpurun_out/ ncu artefacts into committed profiles/ summaries.
usage: python tools/summarize_profiles.py ROUND_TAG"""
import collections
import csv
import io
import json
import os
import subprocess
import sys

tag = sys.argv[1] if len(sys.argv) > 1 else "r1"
G, P = "gpurun_out", "profiles"
os.makedirs(P, exist_ok=True)


def launch_list():
    rows = list(csv.reader(open(os.path.join(G, "launches.csv"))))
    hdr = None
    agg = collections.OrderedDict()
    for r in rows:
        if "Kernel Name" in r:
            hdr = r
            continue
        if not hdr or len(r) != len(hdr):
            continue
        d = dict(zip(hdr, r))
        if d["Metric Name"] != "gpu__time_duration.sum":
            continue
        k = d["Kernel Name"]
        v = float(d["Metric Value"].replace(",", ""))
        scale = {"ns": 1e-3, "us": 1.0, "usecond": 1.0, "nsecond": 1e-3, "ms": 1e3}.get(d["Metric Unit"], 1e-3)
        agg.setdefault(k, []).append(v * scale)
    tot = sum(sum(v) for v in agg.values())
    out = []
    for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        out.append({"kernel": k, "launches": len(v), "mean_us": round(sum(v) / len(v), 2),
                    "min_us": round(min(v), 2), "max_us": round(max(v), 2),
                    "share_of_profiled_time": round(sum(v) / tot, 4)})
    return out


KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "l1tex__t_sector_hit_rate.pct", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "launch__occupancy_limit_registers", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
        "smsp__average_warp_latency_per_inst_issued.ratio", "dram__bytes.sum.per_second"]


def full(rep):
    p = os.path.join(G, rep)
    if not os.path.exists(p):
        return []
    txt = subprocess.run(["ncu", "-i", p, "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")]}
        for k in KEYS:
            if k in hdr:
                i = hdr.index(k)
                d[k] = f"{r[i]} {units[i]}".strip()
        res.append(d)
    return res


summary = {"tag": tag, "launch_list": launch_list(),
           "spmv_full": full("prof_spmv.ncu-rep"), "vector_full": full("prof_vec.ncu-rep")}
json.dump(summary, open(os.path.join(P, f"{tag}_ncu_summary.json"), "w"), indent=1)
# dram bytes per SpMV launch (for bench.py roofline.traffic)
tr = {}
for d in summary["spmv_full"]:
    try:
        rd, ru = d["dram__bytes_read.sum"].split()
        wr, wu = d["dram__bytes_write.sum"].split()
        mul = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
        tr = {"hpccg128": {"dram_bytes_per_launch": float(rd) * mul[ru] + float(wr) * mul[wu],
                           "kernel": d["kernel"], "source": f"profiles/{tag}_ncu_summary.json"}}
    except Exception:
        pass
if tr:
    json.dump(tr, open(os.path.join(P, "spmv_traffic.json"), "w"), indent=1)
for f in ["bench.json", "launches.csv", "smi.txt"]:
    if os.path.exists(os.path.join(G, f)):
        with open(os.path.join(G, f)) as src, open(os.path.join(P, f"{tag}_{f}"), "w") as dst:
            dst.write(src.read())
print(json.dumps(summary["launch_list"][:8], indent=1))
print(json.dumps(summary["spmv_full"], indent=1))
print(json.dumps(summary["vector_full"], indent=1))
