"""Instructions and warp-stall samples of an `ncu --import-source on` capture, summed over source
line ranges of csrc/kernels.cu (the code regions of a kernel: product iteration, hash insert,
sort, ...): python tools/ncu_regions.py rep.ncu-rep FIRST:LAST:name ...  (lines of the profiled
source; lines of other files count as "headers")."""
import csv, io, subprocess, sys
rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
ranges = [(int(a), int(b), n) for a, b, n in (x.split(":") for x in sys.argv[2:])]
agg = {n: [0, 0] for _, _, n in ranges}; agg["other kernels.cu"] = [0, 0]; agg["headers"] = [0, 0]; tot = [0, 0]
fname = None; hdr = None
for r in rows:
    if r and r[0] in ("File Name", "File Path"):
        fname = r[1]; hdr = None; continue
    if r and r[0] == "Line No" and len(r) > 3:
        hdr = r; ie, isamp = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)"); continue
    if hdr is None: continue
    try:
        ln = int(r[0]); ins, smp = int(r[ie]), int(r[isamp])
    except (ValueError, IndexError):
        continue
    tot[0] += ins; tot[1] += smp
    if not fname.endswith("kernels.cu"):
        agg["headers"][0] += ins; agg["headers"][1] += smp; continue
    for a, b, n in ranges:
        if a <= ln <= b:
            agg[n][0] += ins; agg[n][1] += smp; break
    else:
        agg["other kernels.cu"][0] += ins; agg["other kernels.cu"][1] += smp
for n, (i, s) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"{n:28s} inst {100*i/tot[0]:5.1f}%  stall-samples {100*s/tot[1]:5.1f}%")
