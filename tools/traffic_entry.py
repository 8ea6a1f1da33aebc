"""Write one profiles/traffic.json entry from an ncu --set full digest (tools/ncu_summary.py output):
the DRAM bytes of that launch (dram__bytes_read.sum + dram__bytes_write.sum), stamped with the
digest of the kernel sources it was measured on, so that bench.py reports it only for the same code.

usage: python tools/traffic_entry.py DIGEST.md KEY ALG_BYTES_PER_LAUNCH "source description"
  KEY = <kernel>@config<i> (bench.py looks up f"{dominant kernel}@config{--config}")"""
import json
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from bench import source_digest  # noqa: E402

md, key, alg, src = sys.argv[1], sys.argv[2], float(sys.argv[3]), sys.argv[4]
txt = open(md).read()


def metric(name):
    m = re.search(r"\| " + re.escape(name) + r" \| ([0-9.,]+) \| ([^|]*)\|", txt)
    v = float(m.group(1).replace(",", ""))
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "us": 1, "ms": 1e3}.get(m.group(2).strip(), 1)
    return v * scale


dram = metric("dram__bytes_read.sum") + metric("dram__bytes_write.sum")
stalls = re.findall(r"- (\w+)_per_issue_active.ratio: ([0-9.]+)", txt)
top = ", ".join(f"{k} {float(v):.1f}" for k, v in stalls[:3])
entry = {"dram_bytes_per_launch": dram, "alg_bytes_per_launch": alg, "traffic_over_alg": dram / alg,
         "ncu_duration_us": metric("gpu__time_duration.sum"),
         "binding_unit": (f"SM {metric('sm__throughput.avg.pct_of_peak_sustained_elapsed'):.0f} %, LSU "
                          f"{metric('l1tex__data_pipe_lsu_wavefronts.sum.pct_of_peak_sustained_elapsed'):.0f} %; "
                          f"top stalls per issue: {top}"),
         "source": src, "source_digest": source_digest()}
path = os.path.join(ROOT, "profiles", "traffic.json")
d = json.load(open(path)) if os.path.exists(path) else {}
d[key] = entry
json.dump(d, open(path, "w"), indent=1)
print(key, json.dumps(entry, indent=1))
