#!/bin/bash
# Queue-capacity sweep (lu_sym_opts.queue_capacity): QS per config in CFGS (under gpurun).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
for c in ${CFGS:-2 5}; do for q in ${QS:-256 384 512 1024}; do
  timeout 900 python bench.py --config $c --steps ${STEPS:-5} --warmup 2 --no-cpu-baseline --no-e2e --queue-capacity $q 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    if l.startswith('{'):
        d = json.loads(l); print('cfg$c q $q', '%.3f ms/step' % d['ms_per_step'], 'count %.3f' % d['phases_ms']['count'], 'rows', d['plan']['rows_in_flight'], 'spills', d['plan']['spills'])
"
done; done
