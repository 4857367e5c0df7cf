cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
cp abvariants/liblusym_old.so /tmp/ 2>/dev/null
L=paper_conf_ppopp_xia0ar23_b200/lib
AB_CASES=2:0:0,5:250000:0,4:1040000:0,1:0:0,3:0:0 REPS=3 timeout 1500 python scripts/ab_count.py $L/liblusym.so abvariants/liblusym_prev.so > gpurun_out/ab_swzrt.log 2>&1
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/t_swz.log 2>&1; echo rc=$? >> gpurun_out/t_swz.log
