cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
python -c "
import __graft_entry__ as g
g.build_variant('ldcg', {'LUSYM_MERGE_LDCG': 1})
g.build_variant('ku1', {'LUSYM_MERGE_KU': 1})
g.build_variant('ku2', {'LUSYM_MERGE_KU': 2})
" > gpurun_out/bv.log 2>&1
V=paper_conf_ppopp_xia0ar23_b200/lib/variants
for r in 1 2; do
  for hd in 0 2; do
  echo "base head=$hd" >> gpurun_out/mtail2.log; LUSYM_MERGE_GRID_HEAD=$hd python scripts/merge_stats.py >> gpurun_out/mtail2.log 2>&1
  for v in ldcg ku1 ku2; do echo "$v head=$hd" >> gpurun_out/mtail2.log; LUSYM_MERGE_GRID_HEAD=$hd LUSYM_LIB=$V/liblusym_$v.so python scripts/merge_stats.py >> gpurun_out/mtail2.log 2>&1; done
  done
done
