# cluster tail: new members hashed over the ranks (LUSYM_MERGE_HASH=1, default) vs kept local
cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "deferred or cfg3_full" > gpurun_out/t_mhash.log 2>&1; echo "rc=$?" >> gpurun_out/t_mhash.log
python -c "import __graft_entry__ as g; g.build_variant('mhash0', {'LUSYM_MERGE_HASH': 0}); g.build_variant('mprof', {'LUSYM_MERGE_PROF': 1})" > gpurun_out/bv.log 2>&1
V=paper_conf_ppopp_xia0ar23_b200/lib/variants
for r in 1 2; do
  python scripts/merge_stats.py >> gpurun_out/mhash.log 2>&1
  LUSYM_LIB=$V/liblusym_mhash0.so python scripts/merge_stats.py >> gpurun_out/mhash.log 2>&1
done
LUSYM_LIB=$V/liblusym_mprof.so python scripts/merge_stats.py > gpurun_out/mprof.log 2>&1
