"""D2H of C2's output in 9 chunk copies whose boundaries are rounded to 32 elements (the
pipeline's heads), 4 KB, 64 KB or 2 MB of the value array; plus 2 and 3 groups.  Pinned torch
host arrays, best of 5, GB/s of 12 B per nonzero.  Diagnostic for the box-dependent multi-copy
penalty."""
import json
import torch

dev = torch.device("cuda", 0)
Z = 254_840_104
cs = torch.cuda.Stream()
dcol = torch.empty(Z, dtype=torch.int32, device=dev)
dval = torch.empty(Z, dtype=torch.float64, device=dev)
col = torch.empty(Z, dtype=torch.int32, pin_memory=True)
val = torch.empty(Z, dtype=torch.float64, pin_memory=True)


def timed(bounds, reps=5):
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


def groups(k, align_elems):
    return [Z * i // k // align_elems * align_elems for i in range(k)] + [Z]


out = {"val_ptr_mod_2MB": val.data_ptr() % (2 << 20), "col_ptr_mod_2MB": col.data_ptr() % (2 << 20)}
out["one_copy"] = timed([0, Z])
for k in (2, 3, 9):
    for name, al in (("32el", 32), ("4KB", 4096 // 4), ("64KB", 65536 // 4), ("2MB", (2 << 20) // 4)):
        out[f"{k}_groups_{name}"] = timed(groups(k, al))
out["one_copy_again"] = timed([0, Z])
print(json.dumps(out))
