"""Host-link duplex probe (diagnostic): D2H alone, H2D alone, and both at once on two streams
(pinned host buffers, copy engines only).  Tells whether the H2D of the operands can hide under
the D2H of C in the e2e step."""
import json, torch
dev = torch.device("cuda", 0)
n_d2h, n_h2d = 3 << 30, 686 << 20
dsrc = torch.empty(n_d2h, dtype=torch.uint8, device=dev); dsrc.fill_(1)
hdst = torch.empty(n_d2h, dtype=torch.uint8, pin_memory=True)
hsrc = torch.empty(n_h2d, dtype=torch.uint8, pin_memory=True); hsrc.fill_(2)
ddst = torch.empty(n_h2d, dtype=torch.uint8, device=dev)
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
def ev():
    return torch.cuda.Event(enable_timing=True)
out = {}
for rep in range(3):
    for mode in ("d2h", "h2d", "both"):
        torch.cuda.synchronize()
        a0, a1, b0, b1 = ev(), ev(), ev(), ev()
        if mode in ("d2h", "both"):
            with torch.cuda.stream(s1):
                a0.record(s1); hdst.copy_(dsrc, non_blocking=True); a1.record(s1)
        if mode in ("h2d", "both"):
            with torch.cuda.stream(s2):
                b0.record(s2); ddst.copy_(hsrc, non_blocking=True); b1.record(s2)
        torch.cuda.synchronize()
        r = {}
        if mode in ("d2h", "both"):
            r["d2h_ms"] = a0.elapsed_time(a1); r["d2h_GBps"] = n_d2h / r["d2h_ms"] / 1e6
        if mode in ("h2d", "both"):
            r["h2d_ms"] = b0.elapsed_time(b1); r["h2d_GBps"] = n_h2d / r["h2d_ms"] / 1e6
        out[mode] = r
# paced: the D2H in 16 pieces; H2D piece k starts when D2H piece k starts (the H2D spread over
# the whole D2H instead of bunched at its start)
K = 16
for rep in range(3):
    torch.cuda.synchronize()
    a0, a1, b1 = ev(), ev(), ev()
    a0.record(s1)
    for k in range(K):
        e = torch.cuda.Event()
        e.record(s1)
        s2.wait_event(e)
        with torch.cuda.stream(s1):
            hdst[k * n_d2h // K:(k + 1) * n_d2h // K].copy_(dsrc[k * n_d2h // K:(k + 1) * n_d2h // K], non_blocking=True)
        with torch.cuda.stream(s2):
            ddst[k * n_h2d // K:(k + 1) * n_h2d // K].copy_(hsrc[k * n_h2d // K:(k + 1) * n_h2d // K], non_blocking=True)
    a1.record(s1); b1.record(s2)
    torch.cuda.synchronize()
    out["paced"] = {"d2h_ms": a0.elapsed_time(a1), "h2d_end_ms": a0.elapsed_time(b1)}
    out["paced"]["d2h_GBps"] = n_d2h / out["paced"]["d2h_ms"] / 1e6
print(json.dumps(out))
