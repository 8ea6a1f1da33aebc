#!/bin/bash
# One GPU call for the round's evidence (under gpurun): GPU suite (incl. the checked library), bench
# lines (C3 headline with cpu baseline, C2), the ncu launch list of a C3 bench step and full captures
# of the C3 CTA-tier kernels.  usage: bash tools/final_gpu.sh TAG
TAG=${1:-final}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv > gpurun_out/smi_$TAG.txt 2>&1
timeout 1800 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/gputest_$TAG.log 2>&1; echo "gputest rc=$? $(tail -1 gpurun_out/gputest_$TAG.log)"
timeout 900 python bench.py > gpurun_out/bench_c3_$TAG.log 2>&1; echo "bench c3 rc=$?"; tail -1 gpurun_out/bench_c3_$TAG.log | python tools/bench_brief.py c3
timeout 600 python bench.py --config 1 > gpurun_out/bench_c2_$TAG.log 2>&1; echo "bench c2 rc=$?"; tail -1 gpurun_out/bench_c2_$TAG.log | python tools/bench_brief.py c2
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref_$TAG.log 2>&1; echo "ref rc=$? $(tail -1 gpurun_out/bench_ref_$TAG.log | cut -c1-300)"
LAUNCHES=1 bash tools/prof_c3.sh $TAG num_b sym_b
for K in num_b sym_b; do grep -E "gpu__time_duration|dram__bytes|sm__throughput" gpurun_out/ncu_${K}_$TAG.md; done
