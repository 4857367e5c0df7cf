cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build_variant('pfgb', {'LUSYM_PREFETCH_GB': 1})" > gpurun_out/bv.log 2>&1
L=paper_conf_ppopp_xia0ar23_b200/lib
AB_CASES=3:0:0 REPS=4 timeout 1500 python scripts/ab_count.py $L/liblusym.so $L/variants/liblusym_pfgb.so > gpurun_out/ab_pfgb.log 2>&1
