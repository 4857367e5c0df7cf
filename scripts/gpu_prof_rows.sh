cd "${GRAFT_REPO_ROOT:-/root/repo}"; mkdir -p gpurun_out
python scripts/profile_rows.py 4 1184 > gpurun_out/rows4.log 2>&1
python scripts/profile_rows.py 4 1184 512 >> gpurun_out/rows4.log 2>&1
python scripts/profile_rows.py 3 148 >> gpurun_out/rows4.log 2>&1
python scripts/profile_rows.py 3 148 256 >> gpurun_out/rows4.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:fill2_kernel -c 1 -f -o gpurun_out/fill2_cfg4top python scripts/profile_rows.py 4 296 > gpurun_out/ncu4.log 2>&1
cat gpurun_out/rows4.log
