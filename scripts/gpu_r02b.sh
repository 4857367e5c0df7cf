# round 2, session 2: e2e after the handle fix, per-function ncu breakdown of cfg2 / cfg5,
# sanitizers over the async BFS knobs
cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out/r02b /tmp/prof
O=gpurun_out/r02b
timeout 600 python bench.py --steps 5 --warmup 3 --per-config "" --no-numeric > $O/bench_cfg2.log 2>&1; echo "rc=$?" >> $O/bench_cfg2.log
N="ncu --set full --import-source on --clock-control none -k fill2_kernel"
timeout 600 $N --launch-count 1 -o /tmp/prof/c2 python scripts/prof_count.py 2 > $O/p_cfg2.log 2>&1
timeout 600 $N --launch-skip 1 --launch-count 1 -o /tmp/prof/c5 python scripts/prof_count.py 5 250000 0 > $O/p_cfg5.log 2>&1
for c in c2 c5; do
  python scripts/ncu_funcs.py /tmp/prof/$c.ncu-rep > $O/funcs_$c.txt 2>&1
  python scripts/ncu_hot.py /tmp/prof/$c.ncu-rep 60 > $O/hot_$c.txt 2>&1
  ncu -i /tmp/prof/$c.ncu-rep --page source --csv --print-source cuda > $O/src_$c.csv 2>/dev/null
done
for t in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $t python scripts/sanitize.py > $O/san_$t.log 2>&1; echo "rc=$?" >> $O/san_$t.log
done
