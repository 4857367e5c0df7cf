#!/bin/bash
# Full check of the current tree on one B200 (under gpurun): smoke, GPU parity tests, bench lines
# for the configs in CFGS, and (PROF=1) the cfg2 launch list + ncu --set full of fill2.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.used --format=csv > gpurun_out/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
if [ -z "$NOTEST" ]; then
timeout ${TEST_TIMEOUT:-1200} python -m pytest tests -x -q -m "gpu" ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
fi
timeout 600 python bench.py > gpurun_out/bench_cfg2.log 2>&1; echo "rc=$?" >> gpurun_out/bench_cfg2.log
for c in ${CFGS}; do
  timeout 900 python bench.py --config $c --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_cfg$c.log 2>&1; echo "rc=$?" >> gpurun_out/bench_cfg$c.log
done
if [ -n "$PROF" ]; then bash scripts/profile_round.sh; fi
tail -n 3 gpurun_out/smoke.log gpurun_out/pytest_gpu.log
