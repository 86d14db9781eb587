"""gpurun_out/prof_f1f4.ncu-rep (tools/f_ncu.py under ncu --set full
--graph-profiling graph) -> profiles/r1_ncu_f1f4.json: DRAM bytes per
iteration of the fused tridiagonal CG (difference of a 5- and a 1-iteration
solve graph, / 4) and per LBM step launch (cold-cache replay: the step's
writes mostly stay in L2, so DRAM writes undercount them)."""
import csv
import io
import json
import subprocess
import sys

tag = sys.argv[1] if len(sys.argv) > 1 else "r1"
M = "gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum"
txt = subprocess.run(["ncu", "-i", "gpurun_out/prof_f1f4.ncu-rep", "--page", "raw", "--csv",
                      "--metrics", M], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
hdr, units = rows[0], rows[1]
scale = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}


def val(r, k):
    i = hdr.index(k)
    return float(r[i].replace(",", "")) * scale.get(units[i], 1.0)


graphs = [r for r in rows[2:] if "graph" in r[hdr.index("Kernel Name")]]
lbm = [r for r in rows[2:] if "lbm_pull_kernel" in r[hdr.index("Kernel Name")]]
out = {"source": "ncu --set full --graph-profiling graph (tools/f_ncu.py), cold-cache replays"}
if len(graphs) >= 2:
    n = 100_000_000
    rd = (val(graphs[1], "dram__bytes_read.sum") - val(graphs[0], "dram__bytes_read.sum")) / 4
    wr = (val(graphs[1], "dram__bytes_write.sum") - val(graphs[0], "dram__bytes_write.sum")) / 4
    out["tridiag"] = {"dram_bytes_per_iteration": rd + wr, "read": rd, "write": wr,
                      "algorithmic_bytes_per_iteration": 112.0 * n,
                      "how": "(5-iteration solve graph - 1-iteration solve graph) / 4, fused variant"}
if lbm:
    rd = sum(val(r, "dram__bytes_read.sum") for r in lbm) / len(lbm)
    wr = sum(val(r, "dram__bytes_write.sum") for r in lbm) / len(lbm)
    out["lbm"] = {"dram_bytes_per_launch": rd + wr, "read": rd, "write": wr,
                  "algorithmic_bytes_per_launch": 144.0 * 998 * 998,
                  "how": "mean over %d lbm_pull_kernel launches at 1000^2; writes left in L2 at "
                         "kernel end are not counted by a cold-cache replay" % len(lbm)}
json.dump(out, open(f"profiles/{tag}_ncu_f1f4.json", "w"), indent=1)
print(json.dumps(out, indent=1))
