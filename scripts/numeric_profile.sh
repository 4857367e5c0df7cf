#!/bin/bash
# Numeric phase on one B200 (under gpurun): GPU tests, timing, ncu launch list + one full capture.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 900 python -m pytest tests -q -m gpu ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
timeout 400 python scripts/numeric_time.py > gpurun_out/numeric_time.log 2>&1; cat gpurun_out/numeric_time.log
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv \
    --log-file gpurun_out/numeric_launches_cfg1.csv python scripts/numeric_time.py "cfg1 lap2d_k64" > gpurun_out/numeric_launches.log 2>&1
timeout 400 ncu --set full --clock-control none --import-source on -k k_update_level -s 6000 -c 1 \
    -o gpurun_out/ncu_numeric_lap3d24 -f python scripts/numeric_time.py lap3d_k24 > gpurun_out/ncu_numeric.log 2>&1
tail -3 gpurun_out/ncu_numeric.log
