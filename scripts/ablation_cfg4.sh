#!/bin/bash
# cfg4 subset of the design ablation (the chunking/row-class rows of SURVEY 8(f1)); under gpurun.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
for v in "0:B200 design (default)" "128:ONE_CLASS (Alg.3 single chunk size)" \
         "2048:PAPER_CHUNKS (Alg.4: L/(6n)-row launches)" "2176:PAPER_CHUNKS|ONE_CLASS (Alg.3 launches)" \
         "8192:MANAGED_PREFETCH (UM scratch, prefetched)"; do
  f=${v%%:*}; label=${v#*:}
  timeout 900 python bench.py --config 4 --steps ${STEPS:-1} --warmup 1 --no-cpu-baseline --no-e2e \
      --flags $f 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    if l.startswith('{'):
        d = json.loads(l); p = d['phases_ms']
        print('cfg4 %-44s step %10.2f ms  count %10.2f  emit %8.2f  levelize %8.2f  rows/flight %5d classes? %s launches %s' % (
            '$label', d['ms_per_step'], p['count'], p['emit'], p['levelize'], d['plan']['rows_in_flight'], d['plan'].get('row_classes', '-'), d['gpu_launches']))
        break
else:
    print('cfg4 %-44s FAILED' % '$label')
"
done
