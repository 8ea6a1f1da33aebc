#!/bin/bash
# One GPU round trip for a kernel change: parity tests, bench line, ncu of the two W kernels.
# usage (under gpurun): bash tools/gpu_perf.sh TAG
TAG=${1:-x}
mkdir -p gpurun_out
python -m pytest tests/test_gpu_parity.py tests/test_gpu_panels.py -x -q -p no:cacheprovider > gpurun_out/parity_$TAG.log 2>&1
echo "parity rc=$? $(tail -1 gpurun_out/parity_$TAG.log)"
python bench.py --no-cpu > gpurun_out/bench_$TAG.log 2>&1
tail -1 gpurun_out/bench_$TAG.log | python -c "import json,sys;d=json.loads(sys.stdin.read());r=d['roofline'];print('bench',round(d['value'],2),'GF/s',round(d['ms_per_step'],2),'ms e2e',round(d['e2e']['value'],2),'link',round(d['d2h']['host_link_GBps'],1),'frac_link',round(d['d2h']['frac_of_link_bound'],3),'dom',r['kernel'],'frac',round(r['frac'],4),{k:round(v,2) for k,v in r['per_kernel_ms_per_step'].items()})"
for K in num_w sym_w; do
  ncu --set full --clock-control none --import-source on -k regex:k_$K --launch-skip 12 --launch-count 1 -o gpurun_out/prof_${K}_$TAG python tools/pipe_once.py > gpurun_out/ncu_${K}_$TAG.log 2>&1
  python tools/ncu_summary.py gpurun_out/prof_${K}_$TAG.ncu-rep > gpurun_out/ncu_${K}_$TAG.md 2>&1
  grep -E "gpu__time_duration|dram__bytes|sm__throughput|\| inst_executed|bank_conflicts|lsu_wavefronts|spilling" gpurun_out/ncu_${K}_$TAG.md
done
