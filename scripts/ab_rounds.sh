# A/B on B200: the working tree (LUSYM_ROUNDS=1) against a variant build with LUSYM_ROUNDS=0
cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build_variant('${VNAME:-rounds0}', {'${VKEY:-LUSYM_ROUNDS}': ${VVAL:-0}})" > gpurun_out/ab_build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "knobs or cfg1_full or cfg2_full or stats_are" > gpurun_out/t_ab.log 2>&1; echo "rc=$?" >> gpurun_out/t_ab.log
AB_CASES=${AB_CASES:-2:0:0,5:250000:0,4:1040000:0,1:0:0,3:0:0} REPS=${REPS:-2} timeout 1500 python scripts/ab_count.py paper_conf_ppopp_xia0ar23_b200/lib/liblusym.so paper_conf_ppopp_xia0ar23_b200/lib/variants/liblusym_${VNAME:-rounds0}.so > gpurun_out/ab_${VNAME:-rounds0}.log 2>&1
