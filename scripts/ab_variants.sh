#!/bin/bash
# A/B the default library against lib/variants/*.so on one config (under gpurun).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
CFG=${CFG:-2}
STEPS=${STEPS:-5}
for lib in paper_conf_ppopp_xia0ar23_b200/lib/liblusym.so paper_conf_ppopp_xia0ar23_b200/lib/variants/*.so; do
  for rep in 1 2; do
    LUSYM_LIB=$PWD/$lib timeout 600 python bench.py --config $CFG --steps $STEPS --warmup 2 \
        --no-cpu-baseline --no-e2e $BENCH_ARGS 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    if l.startswith('{'):
        d = json.loads(l)
        print('$(basename $lib)', 'cfg$CFG', '%.3f ms/step' % d['ms_per_step'],
              'count %.3f' % d['phases_ms']['count'], 'emit %.3f' % d['phases_ms']['emit'], 'rows', d['plan']['rows_in_flight'])
"
  done
done
