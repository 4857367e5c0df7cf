#!/bin/bash
# threads-per-row sweep (every class forced to the same CTA size), under gpurun
cd "${GRAFT_REPO_ROOT:-/root/repo}"
for c in ${CFGS:-3 5 4}; do
  for t in ${TPRS:-0 128 256 512 1024}; do
    steps=${STEPS:-3}; [ "$c" = 4 ] && steps=1
    timeout 900 python bench.py --config $c --steps $steps --warmup 1 --no-cpu-baseline --no-e2e \
        --threads-per-row $t 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    if l.startswith('{'):
        d = json.loads(l)
        print('cfg$c tpr $t', '%.3f ms/step' % d['ms_per_step'], 'count %.3f' % d['phases_ms']['count'],
              'rows', d['plan']['rows_in_flight'], 'nt', d['plan']['threads_per_row'], 'classes', d['plan']['row_classes'], flush=True)
    elif 'Error' in l: print('cfg$c tpr $t', l.strip()[:200])
"
  done
done
