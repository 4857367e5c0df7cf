#!/bin/bash
# Round-end measurement pass on one B200 (under gpurun): GPU tests, smoke, bench lines for all
# BASELINE configs, the reference arm, the cfg2 launch list and ncu captures.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.used --format=csv > gpurun_out/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1200 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench_cfg2.log 2>&1; echo "rc=$?" >> gpurun_out/bench_cfg2.log
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_reference_cfg2.log 2>&1; echo "rc=$?" >> gpurun_out/bench_reference_cfg2.log
timeout 300 python bench.py --config 1 > gpurun_out/bench_cfg1.log 2>&1; echo "rc=$?" >> gpurun_out/bench_cfg1.log
for c in 3 5 4; do
  timeout 1200 python bench.py --config $c --steps 3 --warmup 3 --e2e-steps 1 > gpurun_out/bench_cfg$c.log 2>&1; echo "rc=$?" >> gpurun_out/bench_cfg$c.log
done
CFG=2 bash scripts/profile_round.sh > gpurun_out/profile_round.log 2>&1
tail -n 3 gpurun_out/smoke.log gpurun_out/pytest_gpu.log
timeout 400 python scripts/numeric_time.py > gpurun_out/numeric_time.log 2>&1
