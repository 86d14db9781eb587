"""Record the GPU box's properties (first-call checklist)."""
import json
import os
import subprocess

import torch

out = {}
p = torch.cuda.get_device_properties(0)
out["name"] = p.name
out["sm_count"] = p.multi_processor_count
out["total_mem_gb"] = p.total_memory / 1e9
out["l2_bytes"] = getattr(p, "L2_cache_size", None)
out["cc"] = f"{p.major}.{p.minor}"
out["nproc"] = os.cpu_count()
try:
    out["lscpu_model"] = [l for l in subprocess.run(["lscpu"], capture_output=True, text=True).stdout.splitlines() if "Model name" in l]
except Exception:
    pass
try:
    out["nvidia_smi"] = subprocess.run(["nvidia-smi", "--query-gpu=name,clocks.max.sm,clocks.max.mem,power.limit,memory.total", "--format=csv"], capture_output=True, text=True).stdout
except Exception:
    pass
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/box.json", "w"), indent=1)
print(json.dumps(out))
