"""Per-source-line digest of an ncu --import-source capture (instructions executed, stall samples,
shared wavefronts): python tools/ncu_lines.py rep.ncu-rep [top]"""
import csv, io, subprocess, sys
rep = sys.argv[1]; top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[2]
ix = {h: i for i, h in enumerate(hdr) if h not in ("Source",)}
ie, isamp, iw = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("L1 Wavefronts Shared")
lines = []
tot_i = tot_s = 0
for r in rows[3:]:
    if len(r) > max(ie, isamp, iw) and r[0] not in ("", "Line No"):
        try:
            ins, smp, wf = int(r[ie]), int(r[isamp]), int(r[iw])
        except ValueError:
            continue
        lines.append((ins, smp, wf, r[0], r[1][:90]))
        tot_i += ins; tot_s += smp
lines.sort(reverse=True)
print(f"total warp instructions {tot_i}, stall samples {tot_s}")
print(f"{'inst':>10} {'%':>5} {'samples%':>8} {'smem_wf':>9}  line  source")
for ins, smp, wf, ln, src in lines[:top]:
    print(f"{ins:>10} {100*ins/max(tot_i,1):5.1f} {100*smp/max(tot_s,1):8.1f} {wf:>9}  {ln:>4}  {src}")
