cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build_variant('swz0', {'LUSYM_SWZ': 0})" > gpurun_out/bv.log 2>&1
L=paper_conf_ppopp_xia0ar23_b200/lib
AB_CASES=2:0:0,5:250000:0,4:1040000:0,1:0:0 REPS=3 timeout 1500 python scripts/ab_count.py $L/liblusym.so $L/variants/liblusym_swz0.so > gpurun_out/ab_swz.log 2>&1
