cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build_variant('kw0', {'LUSYM_KAHN_WARP_MAX': 0}); g.build_variant('kw64', {'LUSYM_KAHN_WARP_MAX': 64})" > gpurun_out/bv.log 2>&1
V=paper_conf_ppopp_xia0ar23_b200/lib/variants
for r in 1 2; do for c in 3 2 4; do for rule in u glu3; do
  echo "kw16" >> gpurun_out/ab_kwarp.log; timeout 300 python scripts/lev_time.py $c $rule >> gpurun_out/ab_kwarp.log 2>&1
  echo "kw0" >> gpurun_out/ab_kwarp.log; LUSYM_LIB=$V/liblusym_kw0.so timeout 300 python scripts/lev_time.py $c $rule >> gpurun_out/ab_kwarp.log 2>&1
  echo "kw64" >> gpurun_out/ab_kwarp.log; LUSYM_LIB=$V/liblusym_kw64.so timeout 300 python scripts/lev_time.py $c $rule >> gpurun_out/ab_kwarp.log 2>&1
done; done; done
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "knobs or level or cfg3_full or cfg1 or random or special or fig1 or lap or circuit" > gpurun_out/t_kw.log 2>&1; echo rc=$? >> gpurun_out/t_kw.log
