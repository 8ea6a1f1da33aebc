"""Host-link D2H rate into pinned memory placed on each NUMA node of the GPU box (diagnostic).

For every NUMA node: pin this process to the node's CPUs, allocate a pinned buffer there (first
touch under the node's local policy), and time copy-engine D2H copies into it (CUDA events, best
of 3), both one large copy and 16 back-to-back chunk-sized copies.  Also reports the GPU's own
NUMA node from sysfs.  Prints one JSON line.
"""
import glob
import json
import os
import subprocess

import torch


def cpulist(s):
    out = []
    for part in s.strip().split(","):
        if not part:
            continue
        if "-" in part:
            a, b = part.split("-")
            out.extend(range(int(a), int(b) + 1))
        else:
            out.append(int(part))
    return out


def gpu_numa():
    bus = torch.cuda.get_device_properties(0).pci_bus_id if hasattr(torch.cuda.get_device_properties(0), "pci_bus_id") else None
    try:
        q = subprocess.run(["nvidia-smi", "--query-gpu=pci.bus_id", "--format=csv,noheader"], capture_output=True,
                           text=True).stdout.strip().splitlines()[0].strip()
        bus = q.lower()
    except Exception:  # noqa: BLE001
        pass
    if bus:
        dom, rest = bus.split(":", 1)
        path = f"/sys/bus/pci/devices/{dom[-4:]}:{rest}/numa_node"
        if os.path.exists(path):
            return bus, int(open(path).read().strip())
    return bus, None


def rate(h, src, reps=3, pieces=1):
    s = torch.cuda.Stream()
    best = 1e9
    n = h.numel() // pieces
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        with torch.cuda.stream(s):
            e0.record(s)
            for k in range(pieces):
                h[k * n:(k + 1) * n].copy_(src[k * n:(k + 1) * n], non_blocking=True)
            e1.record(s)
        s.synchronize()
        best = min(best, e0.elapsed_time(e1) / 1e3)
    return h.numel() / best / 1e9


nb = int(os.environ.get("BYTES", str(2 << 30)))
torch.cuda.init()
src = torch.empty(nb, dtype=torch.uint8, device="cuda")
src.fill_(3)
bus, gnode = gpu_numa()
out = {"gpu_bus": bus, "gpu_numa_node": gnode, "nodes": {}}
orig = os.sched_getaffinity(0)
for nd in sorted(glob.glob("/sys/devices/system/node/node[0-9]*")):
    node = int(nd.rsplit("node", 1)[1])
    cpus = set(cpulist(open(os.path.join(nd, "cpulist")).read())) & orig
    if not cpus:
        continue
    os.sched_setaffinity(0, cpus)
    h = torch.empty(nb, dtype=torch.uint8, pin_memory=True)
    h.fill_(1)  # first touch on this node
    out["nodes"][node] = {"cpus": len(cpus), "d2h_one_GBps": rate(h, src), "d2h_16_GBps": rate(h, src, pieces=16)}
    del h
os.sched_setaffinity(0, orig)
h = torch.empty(nb, dtype=torch.uint8, pin_memory=True)
h.fill_(1)
out["default_affinity"] = {"d2h_one_GBps": rate(h, src), "d2h_16_GBps": rate(h, src, pieces=16)}
try:
    out["topo"] = subprocess.run(["nvidia-smi", "topo", "-m"], capture_output=True, text=True).stdout[-800:]
except Exception:  # noqa: BLE001
    pass
print(json.dumps(out))
