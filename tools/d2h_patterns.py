"""D2H throughput under the pipeline's access pattern (diagnostic; writes gpurun_out/d2h_patterns.json)."""
import json, time, torch
s = torch.cuda.Stream(); s2 = torch.cuda.Stream()
N = 3_058_081_248
dcol = torch.empty(N // 12 * 4 // 4, dtype=torch.int32, device="cuda")
dval = torch.empty(N // 12, dtype=torch.float64, device="cuda")
hcol = torch.empty_like(dcol, device="cpu").pin_memory()
hval = torch.empty_like(dval, device="cpu").pin_memory()
res = {}
def timed(fn, reps=3):
    best = 1e9
    for _ in range(reps):
        torch.cuda.synchronize(); e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
        e0.record(s); fn(); e1.record(s); torch.cuda.synchronize(); best = min(best, e0.elapsed_time(e1))
    return best
with torch.cuda.stream(s):
    res["one_copy_each_GBps"] = N / timed(lambda: (hcol.copy_(dcol, non_blocking=True), hval.copy_(dval, non_blocking=True))) / 1e6
    def chunked(nc):
        n = dval.numel(); step = (n + nc - 1) // nc
        def f():
            for c in range(nc):
                a, b = c * step, min(n, (c + 1) * step)
                hcol[a:b].copy_(dcol[a:b], non_blocking=True); hval[a:b].copy_(dval[a:b], non_blocking=True)
        return f
    for nc in (4, 22, 64):
        res[f"chunked_{nc}_GBps"] = N / timed(chunked(nc)) / 1e6
    # with a concurrent memory-heavy kernel on another stream
    big = torch.empty(1 << 30, dtype=torch.float32, device="cuda"); big2 = torch.empty_like(big)
    def busy():
        with torch.cuda.stream(s2):
            for _ in range(40): big2.copy_(big)
    def with_busy():
        busy(); chunked(22)()
    res["chunked_22_with_hbm_copy_kernel_GBps"] = N / timed(with_busy) / 1e6
    a = torch.randn(8192, 8192, dtype=torch.float64, device="cuda")
    def with_gemm():
        with torch.cuda.stream(s2):
            for _ in range(3): a @ a
        chunked(22)()
    res["chunked_22_with_fp64_gemm_GBps"] = N / timed(with_gemm) / 1e6
import os; os.makedirs("gpurun_out", exist_ok=True)
json.dump(res, open("gpurun_out/d2h_patterns.json", "w"), indent=1); print(json.dumps(res, indent=1))
