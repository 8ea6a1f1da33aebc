"""D2H rate of one output's bytes moved as 1 copy vs the pipeline's pattern of a few copies per
array (diagnostic for the output-chunk grouping).  Same pinned destinations, aligned pieces,
no kernels running, best of 5 per variant."""
import json
import torch

dev = torch.device("cuda", 0)
Z = 254_840_104  # C2 nnz
col = torch.empty(Z, dtype=torch.int32, pin_memory=True)
val = torch.empty(Z, dtype=torch.float64, pin_memory=True)
dcol = torch.empty(Z, dtype=torch.int32, device=dev)
dval = torch.empty(Z, dtype=torch.float64, device=dev)
cs = torch.cuda.Stream()


def timed(fn, reps=5):
    best = 1e9
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(cs):
            e0.record(cs)
            fn()
            e1.record(cs)
        cs.synchronize()
        best = min(best, e0.elapsed_time(e1))
    return 12 * Z / best / 1e6


def pieces(bounds, arrays=("col", "val")):
    def f():
        for a, b in zip(bounds[:-1], bounds[1:]):
            if "col" in arrays:
                col[a:b].copy_(dcol[a:b], non_blocking=True)
            if "val" in arrays:
                val[a:b].copy_(dval[a:b], non_blocking=True)
    return f


def geo(first, n):  # group sizes doubling from `first` elements, 32-aligned
    b, x, s = [0], 0, first
    while x < Z:
        x = min(Z, (x + s) // 32 * 32 if x + s < Z else Z)
        b.append(x)
        s *= 2
    return b


out = {}
out["one_copy_per_array"] = timed(pieces([0, Z]))
for k in (4, 9, 16, 36):
    out[f"equal_{k}_groups"] = timed(pieces([Z * i // k // 32 * 32 for i in range(k)] + [Z]))
b9 = [Z * i // 9 // 32 * 32 for i in range(9)] + [Z]


def abba():
    for g, (a, b) in enumerate(zip(b9[:-1], b9[1:])):
        first, second = ((col, dcol), (val, dval)) if g % 2 == 0 else ((val, dval), (col, dcol))
        first[0][a:b].copy_(first[1][a:b], non_blocking=True)
        second[0][a:b].copy_(second[1][a:b], non_blocking=True)


out["9_groups_abba_order"] = timed(abba)
out["9_col_pieces_then_9_val_pieces"] = timed(lambda: (pieces(b9, ("col",))(), pieces(b9, ("val",))()))
out["9_val_pieces_only"] = timed(pieces(b9, ("val",))) * 2 / 3 * 1.0
out["9_col_pieces_only"] = timed(pieces(b9, ("col",))) / 3
cs2 = torch.cuda.Stream()


def two_streams():
    ev = torch.cuda.Event()
    ev.record(cs)
    cs2.wait_event(ev)
    for g, (a, b) in enumerate(zip(b9[:-1], b9[1:])):
        st = cs if g % 2 == 0 else cs2
        with torch.cuda.stream(st):
            col[a:b].copy_(dcol[a:b], non_blocking=True)
            val[a:b].copy_(dval[a:b], non_blocking=True)
    ev2 = torch.cuda.Event()
    ev2.record(cs2)
    cs.wait_event(ev2)


out["9_groups_two_streams"] = timed(two_streams)
n9 = b9[1]
out["9_val_pieces_same_region"] = timed(lambda: [val[:n9].copy_(dval[a:a + n9], non_blocking=True) for a in b9[:-1]]) * 2 / 3 * n9 * 9 / Z
out["doubling_from_7M"] = timed(pieces(geo(7_000_000, 0)))
out["doubling_groups"] = len(geo(7_000_000, 0)) - 1
out["one_copy_per_array_again"] = timed(pieces([0, Z]))
print(json.dumps({k: (round(v, 2) if isinstance(v, float) else v) for k, v in out.items()}))
