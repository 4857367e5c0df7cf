cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build_variant('rq0', {'LUSYM_ROUND_Q': 0})" > gpurun_out/bv.log 2>&1
L=paper_conf_ppopp_xia0ar23_b200/lib
AB_CASES=2:0:0,5:250000:0,4:1040000:0,3:0:0 REPS=3 timeout 1500 python scripts/ab_count.py $L/liblusym.so $L/variants/liblusym_rq0.so > gpurun_out/ab_roundq.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "knobs or cfg2_full or spills" > gpurun_out/t_rq.log 2>&1; echo rc=$? >> gpurun_out/t_rq.log
