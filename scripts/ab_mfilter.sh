cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "deferred or cfg3_full" > gpurun_out/t_mfilter.log 2>&1; echo "rc=$?" >> gpurun_out/t_mfilter.log
for r in 1 2; do for f in 0 1; do echo "NOFILTER=$f" >> gpurun_out/mfilter.log; if [ $f = 1 ]; then LUSYM_MERGE_NOFILTER=1 python scripts/merge_stats.py >> gpurun_out/mfilter.log 2>&1; else python scripts/merge_stats.py >> gpurun_out/mfilter.log 2>&1; fi; done; done
