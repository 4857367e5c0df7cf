# A/B of the asynchronous BFS (bfs_async) on cfg4's heaviest rows, knobs from the environment
cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "knobs or stats_are" > gpurun_out/t_async.log 2>&1; echo "rc=$?" >> gpurun_out/t_async.log
run() { echo "$*" >> gpurun_out/ab_async_cfg4.log; env "$@" timeout 300 python scripts/exp_ranges.py 4 1040000:1048576 >> gpurun_out/ab_async_cfg4.log 2>&1; }
run LUSYM_ASYNC_OCC=0
for k in 8 32; do for sl in 400 1500; do run LUSYM_ASYNC_KEEP=$k LUSYM_ASYNC_SLEEP=$sl; done; done
run LUSYM_ASYNC_OCC=0
