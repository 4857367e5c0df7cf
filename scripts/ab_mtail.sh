# cluster tail variants on cfg3: kU = 8, batched visited loads, both
cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
python -c "
import __graft_entry__ as g
g.build_variant('ku8', {'LUSYM_MERGE_KU': 8})
g.build_variant('mbatch', {'LUSYM_MERGE_BATCH': 1})
g.build_variant('mbatch8', {'LUSYM_MERGE_BATCH': 1, 'LUSYM_MERGE_KU': 8})
g.build_variant('mbatch16', {'LUSYM_MERGE_BATCH': 1, 'LUSYM_MERGE_KU': 16})
" > gpurun_out/bv.log 2>&1
V=paper_conf_ppopp_xia0ar23_b200/lib/variants
for r in 1 2; do
  echo base >> gpurun_out/mtail.log; python scripts/merge_stats.py >> gpurun_out/mtail.log 2>&1
  for v in ku8 mbatch mbatch8 mbatch16; do echo $v >> gpurun_out/mtail.log; LUSYM_LIB=$V/liblusym_$v.so python scripts/merge_stats.py >> gpurun_out/mtail.log 2>&1; done
done
