#!/bin/bash
# ncu evidence for the C3 headline (under gpurun): launch list of one bench step, full captures of
# one mid-step unit of the CTA-tier kernels.  usage: bash tools/prof_c3.sh TAG [kernels...]
TAG=${1:-x}; shift
KS=${@:-num_b sym_b}
mkdir -p gpurun_out
for K in $KS; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_${K}$" --launch-skip 70 --launch-count 1 \
     -o gpurun_out/prof_${K}_$TAG python tools/c3_once.py > gpurun_out/ncu_${K}_$TAG.log 2>&1
  python tools/ncu_summary.py gpurun_out/prof_${K}_$TAG.ncu-rep > gpurun_out/ncu_${K}_$TAG.md 2>&1

done
if [ -n "$LAUNCHES" ]; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3_$TAG.csv \
     python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu > gpurun_out/launches_c3_$TAG.log 2>&1
  python tools/launch_list.py gpurun_out/launches_c3_$TAG.csv "bench.py --steps 1 --warmup 3 --no-e2e --no-cpu" > gpurun_out/launches_c3_$TAG.md
fi
