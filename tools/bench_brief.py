"""Read one bench.py JSON line on stdin and print the key numbers (for sweeps under gpurun)."""
import json, sys
tag = sys.argv[1] if len(sys.argv) > 1 else ""
d = json.loads(sys.stdin.read().strip().splitlines()[-1])
r = d["roofline"]
print(tag, round(d["value"], 2), "GF/s", round(d["ms_per_step"], 2), "ms", "e2e", round(d["e2e"]["value"], 2) if d.get("e2e") else None,
      r["kernel"], "frac", round(r["frac"], 4), "link", round(d["d2h"]["host_link_GBps"], 1),
      {k: v["ms"] for k, v in r["per_kernel"].items()})
