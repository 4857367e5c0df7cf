#!/bin/bash
# Design ablation on B200: each LU_F_* flag switches one B200 design choice back
# to the paper's printed scheme.  Run under gpurun; prints one line per (config, variant).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
run() {  # cfg flags label
  timeout 900 python bench.py --config $1 --steps ${STEPS:-2} --warmup 1 --no-cpu-baseline --no-e2e \
      --flags $2 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    if l.startswith('{'):
        d = json.loads(l); p = d['phases_ms']
        print('cfg$1 %-44s step %10.2f ms  count %10.2f  emit %8.2f  levelize %8.2f  rows/flight %5d classes? %s' % (
            '$3', d['ms_per_step'], p['count'], p['emit'], p['levelize'], d['plan']['rows_in_flight'], d['plan'].get('row_classes', '-')))
        break
else:
    print('cfg$1 %-44s FAILED' % '$3')
"
}
for c in ${CFGS:-2 5 3}; do
  run $c 0   "B200 design (default)"
  run $c 64  "TWO_PASS (symbolic_2 re-traverses)"
  run $c 128 "ONE_CLASS (Alg.3 single chunk size)"
  run $c 2048 "PAPER_CHUNKS (Alg.4: L/(6n)-row launches)"
  run $c 2176 "PAPER_CHUNKS|ONE_CLASS (Alg.3 launches)"
  run $c 2   "NO_BATCH (one threshold at a time)"
  run $c 40  "NO_CONTRACT|NO_PRUNE (plain Alg.5 Kahn)"
  run $c 1   "GLOBAL_BITMAP (visited state in HBM)"
  run $c 4096 "MANAGED (UM scratch, first-touch faults)"
  run $c 8192 "MANAGED_PREFETCH (UM scratch, prefetched)"
  run $c 4097 "MANAGED|GLOBAL_BITMAP (visited state in UM)"
  run $c 2283 "paper as printed (all of the above)"
done
