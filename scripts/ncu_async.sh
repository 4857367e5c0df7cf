# ncu of the one-CTA-per-SM class on cfg4's heaviest rows: level-synchronous BFS vs bfs_async
cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out/async /tmp/prof
N="ncu --set full --import-source on --clock-control none -k fill2_kernel --launch-skip 1 --launch-count 1"
timeout 600 $N -o /tmp/prof/sync python scripts/prof_count.py 4 1046000 0 > gpurun_out/async/sync.log 2>&1
LUSYM_ASYNC_OCC=2 timeout 600 $N -o /tmp/prof/async python scripts/prof_count.py 4 1046000 0 > gpurun_out/async/async.log 2>&1
for v in sync async; do
  python scripts/ncu_hot.py /tmp/prof/$v.ncu-rep 40 > gpurun_out/async/hot_$v.txt 2>&1
  ncu -i /tmp/prof/$v.ncu-rep --page details --csv > gpurun_out/async/details_$v.csv 2>/dev/null
  ncu -i /tmp/prof/$v.ncu-rep --page raw --csv > gpurun_out/async/raw_$v.csv 2>/dev/null
done
