"""Turn gpurun_out/ ncu artefacts into committed profiles/ summaries.

usage: python tools/summarize_profiles.py TAG [WORKLOAD]

Reads gpurun_out/launches.csv (launch list) and gpurun_out/prof_<WORKLOAD>_{cold,warm}.ncu-rep
(`ncu --set full` of the three CG kernels, tools/profile_round.sh) and writes
profiles/<TAG>_ncu_<WORKLOAD>.json: per kernel the DRAM bytes per launch against
its algorithmic bytes (SpMV 12 nnz + 16 n, x/r update 48 n, p update 24 n; DESIGN
sec. 7), cold and warm cache; merges the SpMV's cold-cache DRAM bytes per launch
into profiles/spmv_traffic.json[WORKLOAD] (bench.py roofline.traffic)."""
import collections
import csv
import io
import json
import os
import subprocess
import sys

tag = sys.argv[1] if len(sys.argv) > 1 else "r2"
W = sys.argv[2] if len(sys.argv) > 2 else "hpccg256"
G, P = "gpurun_out", os.environ.get("PROFILES_OUT", "profiles")
os.makedirs(P, exist_ok=True)
DIMS = {"hpccg256": (256, 256, 256), "hpccg128": (128, 128, 128), "hpccg512s": (512, 512, 512),
        "hpccg20": (20, 30, 10)}


def nnz_of(nx, ny, nz):
    return (3 * nx - 2) * (3 * ny - 2) * (3 * nz - 2)


def launch_list():
    p = os.path.join(G, "launches.csv")
    if not os.path.exists(p):
        return []
    rows = list(csv.reader(open(p)))
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
        scale = {"ns": 1e-3, "us": 1.0, "usecond": 1.0, "nsecond": 1e-3, "ms": 1e3,
                 "msecond": 1e3}.get(d["Metric Unit"], 1e-3)
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
MUL = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6,
       "msecond": 1e-3, "second": 1.0, "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1.0}


def num(v):
    x, u = v.split()
    return float(x.replace(",", "")) * MUL.get(u, 1.0)


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


# the x update is deferred into the p update when the CG vectors exceed L2
# (HPCCG_OPT_DEFER_X auto: 256^3 and 512^3): x/r update 24n, p update 40n
DEFER = {"hpccg256": True, "hpccg512s": True, "hpccg128": False, "hpccg20": False}


def per_kernel(rows, n, nnz):
    d = DEFER.get(W, False)
    alg = {"spmv27x2_kernel": 12.0 * nnz + 16.0 * n, "cg_update1_kernel": (24.0 if d else 48.0) * n,
           "cg_pupdate1_kernel": (40.0 if d else 24.0) * n}
    out = {}
    for d in rows:
        name = next((k for k in alg if k in d["kernel"]), None)
        if not name:
            continue
        dram = num(d["dram__bytes_read.sum"]) + num(d["dram__bytes_write.sum"])
        t = num(d["gpu__time_duration.sum"])
        rec = out.setdefault(name, {"kernel": d["kernel"], "launches": []})
        rec["launches"].append({"dram_read": num(d["dram__bytes_read.sum"]),
                                "dram_write": num(d["dram__bytes_write.sum"]),
                                "dram_over_algorithmic": round(dram / alg[name], 4),
                                "duration_us": round(t * 1e6, 2),
                                "algorithmic_GBs": round(alg[name] / t / 1e9, 1),
                                "l2_hit_pct": d.get("lts__t_sector_hit_rate.pct"),
                                "dram_pct_of_peak": d.get("dram__throughput.avg.pct_of_peak_sustained_elapsed"),
                                "registers": d.get("launch__registers_per_thread")})
        rec["algorithmic_bytes"] = alg[name]
    for rec in out.values():
        ls = rec["launches"]
        rec["dram_bytes_per_launch"] = sum(x["dram_read"] + x["dram_write"] for x in ls) / len(ls)
        rec["dram_over_algorithmic"] = round(rec["dram_bytes_per_launch"] / rec["algorithmic_bytes"], 4)
    return out


RING_M = {"hpccg256": 8, "hpccg512s": 8}


def per_ring(rows, n):
    """cg_pupdate_ring_kernel launches K = 1, 2, ... of the first solve:
    algorithmic bytes 16n (K = 1: r -> p), 24n (r, p -> p), (m + 4) 8n at the
    flush (K - 1 divisible by m: r, p, x and m - 1 old p's -> p, x)."""
    m = RING_M.get(W, 0)
    out = []
    for K, d in enumerate((r for r in rows if "cg_pupdate_ring_kernel" in r["kernel"]), start=1):
        flush = K > 1 and (K - 1) % m == 0
        alg = (16.0 if K == 1 else (m + 4) * 8.0 if flush else 24.0) * n
        dram = num(d["dram__bytes_read.sum"]) + num(d["dram__bytes_write.sum"])
        t = num(d["gpu__time_duration.sum"])
        out.append({"K": K, "flush": flush, "algorithmic_bytes": alg, "dram_read": num(d["dram__bytes_read.sum"]),
                    "dram_write": num(d["dram__bytes_write.sum"]), "dram_over_algorithmic": round(dram / alg, 4),
                    "duration_us": round(t * 1e6, 2), "algorithmic_GBs": round(alg / t / 1e9, 1),
                    "l2_hit_pct": d.get("lts__t_sector_hit_rate.pct"),
                    "registers": d.get("launch__registers_per_thread")})
    return out


nx, ny, nz = DIMS[W]
n, nnz = nx * ny * nz, nnz_of(nx, ny, nz)
summary = {"tag": tag, "workload": W, "n": n, "nnz": nnz, "launch_list": launch_list()}
for cache in ("cold", "warm"):
    rows = full(f"prof_{W}_{cache}.ncu-rep")
    summary[f"{cache}_raw"] = rows
    summary[cache] = per_kernel(rows, n, nnz)
    rr = full(f"prof_{W}_ring_{cache}.ncu-rep")
    if rr:
        summary[f"{cache}_ring_raw"] = rr
        summary[f"{cache}_ring"] = per_ring(rr, n)
out = os.path.join(P, f"{tag}_ncu_{W}.json")
json.dump(summary, open(out, "w"), indent=1)
sp = summary.get("cold", {}).get("spmv27x2_kernel")
if sp:
    tp = os.path.join(P, "spmv_traffic.json")
    tr = json.load(open(tp)) if os.path.exists(tp) else {}
    tr[W] = {"dram_bytes_per_launch": sp["dram_bytes_per_launch"], "kernel": sp["kernel"],
             "dram_over_algorithmic": sp["dram_over_algorithmic"], "cache": "cold (ncu default flush)",
             "source": out}
    json.dump(tr, open(tp, "w"), indent=1)
for f in ["launches.csv", "smi.txt"]:
    if os.path.exists(os.path.join(G, f)):
        with open(os.path.join(G, f)) as src, open(os.path.join(P, f"{tag}_{W}_{f}"), "w") as dst:
            dst.write(src.read())
print(json.dumps(summary["launch_list"][:8], indent=1))
for cache in ("cold", "warm"):
    for k, v in summary[cache].items():
        print(cache, k, v["dram_over_algorithmic"], [x["duration_us"] for x in v["launches"]])
    for x in summary.get(f"{cache}_ring", []):
        print(cache, "ring K=%d" % x["K"], x["flush"], x["dram_over_algorithmic"], x["duration_us"], x["algorithmic_GBs"])
