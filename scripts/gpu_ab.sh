#!/bin/bash
# parity tests on the default build, then A/B of default vs lib/variants/*.so on CFGS (under gpurun)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout ${TEST_TIMEOUT:-900} python -m pytest tests -x -q -m "gpu" ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
for c in ${CFGS:-2 5 3}; do CFG=$c STEPS=${STEPS:-5} bash scripts/ab_variants.sh; done > gpurun_out/ab.log 2>&1
cat gpurun_out/ab.log
