cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build_variant('small2048', {'LUSYM_THREADS_PER_SM_SMALL': 2048})" > gpurun_out/bv.log 2>&1
AB_CASES=2:0:0,3:0:0,5:0:0,1:0:0 REPS=3 timeout 1500 python scripts/ab_count.py paper_conf_ppopp_xia0ar23_b200/lib/liblusym.so paper_conf_ppopp_xia0ar23_b200/lib/variants/liblusym_small2048.so > gpurun_out/ab_regs2.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "knobs or cfg2_full or cfg3_full or sparse" > gpurun_out/t_regs2.log 2>&1; echo rc=$? >> gpurun_out/t_regs2.log
