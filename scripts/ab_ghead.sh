cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "deferred or cfg3_full" > gpurun_out/t_ghead.log 2>&1; echo "rc=$?" >> gpurun_out/t_ghead.log
for r in 1 2; do for k in 0 1 2 3 4 6; do echo "HEAD=$k" >> gpurun_out/ghead.log; LUSYM_MERGE_GRID_HEAD=$k python scripts/merge_stats.py >> gpurun_out/ghead.log 2>&1; done; done
