"""Summarise the DIA-27 SpMV ncu captures (tools/gpu_dia.sh) into
profiles/r1_ncu_dia.json and add their DRAM bytes per launch to
profiles/spmv_traffic.json (bench.py's roofline.traffic for --spmv-format dia)."""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRICS = ["dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum",
           "launch__registers_per_thread", "sm__warps_active.avg.pct_of_peak_sustained_active",
           "lts__t_sector_hit_rate.pct", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
           "launch__grid_size"]
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-3, "us": 1, "ms": 1e3}


def read(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--metrics", ",".join(METRICS)],
                         capture_output=True, text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    head, units, data = rows[0], rows[1], rows[2:]
    res = []
    for r in data:
        d = {"kernel": r[head.index("Kernel Name")]}
        for m in METRICS:
            if m in head:
                i = head.index(m)
                v = float(r[i].replace(",", ""))
                d[m] = v * UNIT.get(units[i], 1)
        res.append(d)
    return res


def main(rnd="r1"):
    summ, traffic = {}, json.load(open(os.path.join(ROOT, "profiles", "spmv_traffic.json")))
    for wl, rep, n in [("hpccg128_dia", "prof_spmv_dia", 128 ** 3), ("hpccg256_dia", "prof_spmv_dia256", 256 ** 3)]:
        path = os.path.join(ROOT, "gpurun_out", rep + ".ncu-rep")
        if not os.path.exists(path):
            continue
        launches = read(path)
        dram = sum(x["dram__bytes_read.sum"] + x["dram__bytes_write.sum"] for x in launches) / len(launches)
        summ[wl] = {"launches": launches, "algorithmic_bytes_per_launch": 232.0 * n,
                    "dram_bytes_per_launch": dram, "dram_over_algorithmic": dram / (232.0 * n),
                    "note": "cold cache (ncu default --cache-control all), --clock-control none; units: bytes, us"}
        traffic[wl] = {"dram_bytes_per_launch": dram, "kernel": launches[0]["kernel"],
                       "source": f"profiles/{rnd}_ncu_dia.json"}
    json.dump(summ, open(os.path.join(ROOT, "profiles", f"{rnd}_ncu_dia.json"), "w"), indent=1)
    json.dump(traffic, open(os.path.join(ROOT, "profiles", "spmv_traffic.json"), "w"), indent=1)
    print(json.dumps({k: (v["dram_bytes_per_launch"], v["dram_over_algorithmic"]) for k, v in summ.items()}))


if __name__ == "__main__":
    main(*sys.argv[1:])
