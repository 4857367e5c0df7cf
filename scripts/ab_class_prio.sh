cd "${GRAFT_REPO_ROOT:-/root/repo}"
run() { timeout 900 python bench.py --config $1 --steps ${S:-2} --warmup 1 --no-cpu-baseline --no-e2e --flags $2 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    if l.startswith('{'): d=json.loads(l); print('$3 cfg$1', round(d['ms_per_step'],2), round(d['phases_ms']['count'],2), d['plan']['row_classes'])
"; }
for c in 3 5; do
  run $c 0 "prio+window"; run $c 16384 "prio only"; LUSYM_NO_CLASS_PRIO=1 run $c 0 "window only"
  LUSYM_LIB=$PWD/paper_conf_ppopp_xia0ar23_b200/lib/variants/liblusym_head.so run $c 0 "head"
done
S=1; c=4; run $c 0 "prio+window"; run $c 16384 "prio only"; LUSYM_LIB=$PWD/paper_conf_ppopp_xia0ar23_b200/lib/variants/liblusym_head.so run $c 0 "head"
