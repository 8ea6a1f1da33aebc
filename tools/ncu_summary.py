"""Summarise an `ncu --set full` report (.ncu-rep) into a small JSON/markdown digest for profiles/.

usage: python tools/ncu_summary.py gpurun_out/prof_numw.ncu-rep [--source] > profiles/r01/ncu_numw.md
"""
import csv
import io
import subprocess
import sys

NCU = "/usr/local/cuda/bin/ncu"
KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
    "lts__t_bytes.sum", "l1tex__t_bytes.sum", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed.sum", "smsp__inst_executed.avg.per_cycle_active", "sm__cycles_elapsed.avg",
    "launch__registers_per_thread", "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
    "sm__maximum_warps_per_active_cycle_pct", "launch__grid_size", "launch__block_size",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "smsp__average_warp_latency_issue_stalled",
    "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct",
    "inst_executed", "l1tex__data_pipe_lsu_wavefronts.sum.pct_of_peak_sustained_elapsed",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "sass__inst_executed_register_spilling",
]
STALLS = "smsp__average_warps_issue_stalled_"


def raw(rep):
    out = subprocess.run([NCU, "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {h: (v, u) for h, v, u in zip(hdr, r, units)}
        res.append(d)
    return res


def main():
    rep = sys.argv[1]
    for d in raw(rep):
        name = d.get("Kernel Name", ("?", ""))[0]
        print(f"### {name[:90]}\n")
        print("| metric | value | unit |\n|---|---|---|")
        for k in KEYS:
            if k in d:
                print(f"| {k} | {d[k][0]} | {d[k][1]} |")
        stalls = sorted(((k[len(STALLS):], d[k][0]) for k in d if k.startswith(STALLS) and k.endswith("_per_issue_active.ratio")),
                        key=lambda kv: -float(kv[1].replace(",", "") or 0))
        print("\nTop stall reasons (warps stalled per issue):\n")
        for k, v in stalls[:10]:
            print(f"- {k}: {v}")
        print()
    if "--source" in sys.argv:
        out = subprocess.run([NCU, "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                             capture_output=True, text=True).stdout
        print("\n(source page: %d lines)" % len(out.splitlines()))


if __name__ == "__main__":
    main()
