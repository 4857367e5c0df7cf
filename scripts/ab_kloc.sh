# self-continuation in classes with <= 1 / <= 2 (default) / <= 4 rows per SM (LUSYM_KLOC_OCC)
cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build_variant('kocc1', {'LUSYM_KLOC_OCC': 1}); g.build_variant('kocc4', {'LUSYM_KLOC_OCC': 4})" > gpurun_out/ab_build.log 2>&1
L=paper_conf_ppopp_xia0ar23_b200/lib
AB_CASES=4:0:0,5:0:0 REPS=2 timeout 1500 python scripts/ab_count.py $L/liblusym.so $L/variants/liblusym_kocc1.so $L/variants/liblusym_kocc4.so > gpurun_out/ab_kloc.log 2>&1
