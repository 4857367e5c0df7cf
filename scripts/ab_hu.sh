cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out

V=abvariants/liblusym_old.so
for r in 1 2; do for c in 3 1 2; do for rule in u glu3; do
  echo "new" >> gpurun_out/ab_hu.log; timeout 300 python scripts/lev_time.py $c $rule >> gpurun_out/ab_hu.log 2>&1
  echo "old" >> gpurun_out/ab_hu.log; LUSYM_LIB=$V timeout 300 python scripts/lev_time.py $c $rule >> gpurun_out/ab_hu.log 2>&1
done; done; done
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "knobs or level or cfg3_full or cfg1" > gpurun_out/t_hu.log 2>&1; echo rc=$? >> gpurun_out/t_hu.log
