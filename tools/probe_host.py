"""Box probe: device properties, host resources, pinned host-link bandwidth.

Run under gpurun; writes gpurun_out/probe.json. Measures the D2H/H2D
rate of cudaMemcpyAsync between device memory and pinned host memory
(the host-link peak that S8 of SURVEY §8(a) is judged against) and the
cost of pinning host memory.
"""
import json, os, time, subprocess
import torch

out = {}
p = torch.cuda.get_device_properties(0)
out["device"] = {"name": p.name, "sms": p.multi_processor_count,
                 "total_mem": p.total_memory, "cc": [p.major, p.minor],
                 "l2": getattr(p, "L2_cache_size", None)}
out["ncpu"] = os.cpu_count()
try:
    out["sched_affinity"] = len(os.sched_getaffinity(0))
except Exception:
    pass
with open("/proc/meminfo") as f:
    out["meminfo"] = {l.split(":")[0]: l.split(":")[1].strip() for l in f.readlines()[:5]}
try:
    out["lscpu"] = subprocess.run(["lscpu"], capture_output=True, text=True).stdout
except Exception:
    pass
try:
    out["topo"] = subprocess.run(["nvidia-smi", "topo", "-m"], capture_output=True, text=True).stdout
    out["pcie"] = subprocess.run(["nvidia-smi", "--query-gpu=pcie.link.gen.current,pcie.link.gen.max,pcie.link.width.current,pcie.link.width.max",
                                  "--format=csv"], capture_output=True, text=True).stdout
except Exception:
    pass

res = {}
s = torch.cuda.Stream()
for mb in [16, 64, 256, 1024, 2048]:
    n = mb << 20
    t0 = time.perf_counter()
    h = torch.empty(n, dtype=torch.uint8, pin_memory=True)
    t_pin = time.perf_counter() - t0
    d = torch.empty(n, dtype=torch.uint8, device="cuda")
    d.fill_(1)
    torch.cuda.synchronize()
    for direction in ("d2h", "h2d"):
        best = 1e9
        for it in range(5):
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            with torch.cuda.stream(s):
                e0.record(s)
                if direction == "d2h":
                    h.copy_(d, non_blocking=True)
                else:
                    d.copy_(h, non_blocking=True)
                e1.record(s)
            s.synchronize()
            best = min(best, e0.elapsed_time(e1) / 1e3)
        res[f"{direction}_{mb}MB_GBps"] = n / best / 1e9
    res[f"pin_{mb}MB_s"] = t_pin
    del h, d
# pageable
n = 256 << 20
hp = torch.empty(n, dtype=torch.uint8)
d = torch.empty(n, dtype=torch.uint8, device="cuda")
torch.cuda.synchronize(); t0 = time.perf_counter()
for _ in range(3):
    hp.copy_(d)
torch.cuda.synchronize()
res["d2h_pageable_256MB_GBps"] = 3 * n / (time.perf_counter() - t0) / 1e9
out["hostlink"] = res
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/probe.json", "w"), indent=1)
print(json.dumps(res, indent=1))
print(out["device"], out["ncpu"], out["meminfo"])
