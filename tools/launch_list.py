"""Summarise an ncu launch list (`ncu --metrics gpu__time_duration.sum --csv --log-file X.csv ...`)
into a per-kernel markdown table: launches, total us, share.  usage: python tools/launch_list.py X.csv "cmd" """
import collections
import csv
import sys

path, cmd = sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else ""
rows = [r for r in csv.reader(open(path)) if r]
hdr_i = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
hdr = rows[hdr_i]
ik, iv, im = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Name")
agg = collections.OrderedDict()
for r in rows[hdr_i + 1:]:
    if len(r) <= iv or r[im] != "gpu__time_duration.sum":
        continue
    name = r[ik].split("(")[0].replace("void spg::", "").replace("spg::", "")
    v = float(r[iv].replace(",", ""))
    unit = r[hdr.index("Metric Unit")] if "Metric Unit" in hdr else "nsecond"
    us = v / 1e3 if unit.startswith("n") else v * 1e3 if unit.startswith("m") else v
    a = agg.setdefault(name, [0, 0.0])
    a[0] += 1
    a[1] += us
tot = sum(a[1] for a in agg.values())
print(f"# ncu launch list of `{cmd}`\n")
print("`ncu --metrics gpu__time_duration.sum --clock-control none --csv` -- serialized, cold per-launch times, so only the "
      "SHARES are comparable with the bench's live CUDA-event times.\n")
print("| kernel | launches | total us | share |\n|---|---|---|---|")
for name, (n, us) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    print(f"| {name} | {n} | {us:.1f} | {100 * us / tot:.1f}% |")
