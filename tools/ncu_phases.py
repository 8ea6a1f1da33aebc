"""Per-function / per-lambda breakdown of an ncu --import-source capture of a kernels.cu kernel:
instructions, thread instructions and stall samples grouped by the enclosing function of each
source line (the source file as it was when the capture was built must be the working copy, or give
a git revision).  usage: python tools/ncu_phases.py rep.ncu-rep [git-rev]"""
import collections
import csv
import io
import re
import subprocess
import sys

rep = sys.argv[1]
rev = sys.argv[2] if len(sys.argv) > 2 else None
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
path = "paper_conf_ipps_xia0ar21_b200/csrc/kernels.cu"
src = (subprocess.run(["git", "show", f"{rev}:{path}"], capture_output=True, text=True).stdout if rev
       else open(path).read()).split("\n")
starts = [(i + 1, l.strip()[:72]) for i, l in enumerate(src)
          if re.match(r"^(__device__|__global__|template|struct)", l) or re.search(r"auto \w+ = \[&\]", l)]
cur, hdr = "?", None
agg = collections.defaultdict(lambda: [0, 0, 0])
for r in rows:
    if len(r) > 1 and r[0] == "File Path":
        cur = r[1].split("/")[-1]
        continue
    if len(r) > 1 and r[0] == "Line No":
        hdr = r
        ie, it, isamp = (hdr.index("Instructions Executed"), hdr.index("Thread Instructions Executed"),
                         hdr.index("Warp Stall Sampling (All Samples)"))
        continue
    if hdr is None:
        continue
    try:
        ln, i, t, sm = int(r[0]), int(r[ie]), int(r[it]), int(r[isamp])
    except ValueError:
        continue
    if cur != "kernels.cu":
        key = "(header) " + cur
    else:
        key = max(((s, l) for s, l in starts if s <= ln), default=(0, "?"))
        key = f"{key[0]:5d} {key[1]}"
    a = agg[key]
    a[0] += i
    a[1] += t
    a[2] += sm
TI = sum(v[0] for v in agg.values())
TS = sum(v[2] for v in agg.values())
print(f"total warp instructions {TI}, stall samples {TS}")
print(f"{'inst%':>6} {'smp%':>6} {'thr/inst':>8}  region")
for k, (i, t, sm) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:20]:
    print(f"{100 * i / TI:6.1f} {100 * sm / TS:6.1f} {t / max(i, 1):8.1f}  {k}")
