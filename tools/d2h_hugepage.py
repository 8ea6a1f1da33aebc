"""D2H of C2's output in 9 chunk copies into (a) torch pinned host arrays, (b) host arrays backed by
transparent huge pages (mmap + madvise(MADV_HUGEPAGE), first-touched, then cudaHostRegister),
with one copy per array as the reference.  Diagnostic for the box-dependent multi-copy penalty."""
import ctypes
import json
import mmap

import numpy as np
import torch

dev = torch.device("cuda", 0)
Z = 254_840_104
cs = torch.cuda.Stream()
dcol = torch.empty(Z, dtype=torch.int32, device=dev)
dval = torch.empty(Z, dtype=torch.float64, device=dev)
rt = torch.cuda.cudart()


def huge(nbytes, dtype):
    m = mmap.mmap(-1, nbytes, flags=mmap.MAP_PRIVATE | mmap.MAP_ANONYMOUS)
    m.madvise(mmap.MADV_HUGEPAGE)
    a = np.frombuffer(m, dtype=np.uint8)
    a[::4096] = 0  # first touch
    t = torch.from_numpy(a).view(dtype)
    assert int(rt.cudaHostRegister(t.data_ptr(), nbytes, 0)) == 0
    return t, m


def thp_pages():
    try:
        for ln in open("/proc/meminfo"):
            if ln.startswith("AnonHugePages"):
                return ln.split(":")[1].strip()
    except OSError:
        return None


def timed(col, val, bounds, reps=5):
    best = 1e9
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(cs):
            e0.record(cs)
            for a, b in zip(bounds[:-1], bounds[1:]):
                col[a:b].copy_(dcol[a:b], non_blocking=True)
                val[a:b].copy_(dval[a:b], non_blocking=True)
            e1.record(cs)
        cs.synchronize()
        best = min(best, e0.elapsed_time(e1))
    return round(12 * Z / best / 1e6, 2)


b9 = [Z * i // 9 // 32 * 32 for i in range(9)] + [Z]
out = {}
pc = torch.empty(Z, dtype=torch.int32, pin_memory=True)
pv = torch.empty(Z, dtype=torch.float64, pin_memory=True)
out["pinned_one_copy"] = timed(pc, pv, [0, Z])
out["pinned_9_groups"] = timed(pc, pv, b9)
hc, m1 = huge(4 * Z, torch.int32)
hv, m2 = huge(8 * Z, torch.float64)
out["AnonHugePages"] = thp_pages()
out["thp_one_copy"] = timed(hc, hv, [0, Z])
out["thp_9_groups"] = timed(hc, hv, b9)
out["pinned_9_groups_again"] = timed(pc, pv, b9)
print(json.dumps(out))
