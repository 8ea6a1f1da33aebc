#!/bin/bash
# Sum of per-launch device times (ncu, serialized) of the W kernels over one C2 multiply, per knob
# setting.  usage (under gpurun): bash tools/knob_sweep.sh "ENV1=a ENV2=b" "ENV1=c" ...
mkdir -p gpurun_out
for cfg in "$@"; do
  env $cfg REPS=1 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_(num|sym)_w" --csv \
      --log-file gpurun_out/sweep.csv python tools/pipe_once.py > /dev/null 2>&1
  python - "$cfg" <<'PY'
import csv, sys, collections
rows = list(csv.reader(open("gpurun_out/sweep.csv")))
hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
h = rows[hi]; k = h.index("Kernel Name"); v = h.index("Metric Value"); u = h.index("Metric Unit")
agg = collections.defaultdict(float); n = collections.Counter()
for r in rows[hi + 1:]:
    if len(r) <= v: continue
    x = float(r[v].replace(",", "")); x = x / 1e3 if r[u] == "ns" else x * 1e3 if r[u] == "ms" else x
    name = r[k].split("(")[0].replace("void spg::", "")
    agg[name] += x; n[name] += 1
print(sys.argv[1] or "default", {a: f"{agg[a]/1e3:.3f} ms/{n[a]}" for a in agg})
PY
done
