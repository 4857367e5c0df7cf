cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build_variant('gbl1', {'LUSYM_GB_L1': 1})" > gpurun_out/bv.log 2>&1
L=paper_conf_ppopp_xia0ar23_b200/lib
AB_CASES=3:0:0,2:0:0 REPS=3 timeout 1500 python scripts/ab_count.py $L/liblusym.so $L/variants/liblusym_gbl1.so > gpurun_out/ab_gbl1.log 2>&1
LUSYM_LIB=$L/variants/liblusym_gbl1.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "knobs or cfg3_full or sparse or stats_are or deferred" > gpurun_out/t_gbl1.log 2>&1; echo rc=$? >> gpurun_out/t_gbl1.log
