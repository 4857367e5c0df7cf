cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
python -c "
import __graft_entry__ as g
g.build_variant('kloc3', {'LUSYM_KLOC': 3})
g.build_variant('kloc6', {'LUSYM_KLOC': 6})
" > gpurun_out/bv.log 2>&1
L=paper_conf_ppopp_xia0ar23_b200/lib
AB_CASES=4:851968:0,4:385024:851968 REPS=2 timeout 1500 python scripts/ab_count.py $L/liblusym.so $L/variants/liblusym_kloc3.so $L/variants/liblusym_kloc6.so > gpurun_out/ab_kloc2.log 2>&1
