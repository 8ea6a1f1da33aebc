#!/bin/bash
# Same-box A/B of output-chunk grouping on the C2 bench (alternating runs).
for k in 1 2 3; do
  for v in 0 1; do
    SPGEMM_NO_GROUPS=$v python bench.py --no-cpu --no-e2e --steps 5 > gpurun_out/ab_${v}_${k}.log 2>&1
    tail -1 gpurun_out/ab_${v}_${k}.log | python -c "import json,sys;d=json.loads(sys.stdin.read());x=d['d2h_detail'];print('no_groups=$v', round(d['value'],2), round(d['ms_per_step'],2), 'probe', round(d['d2h']['host_link_GBps'],1), 'busy_rate', round(x['rate_while_busy_GBps'],1), 'copies', x['copies'])"
  done
done
