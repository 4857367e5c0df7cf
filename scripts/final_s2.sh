#!/bin/bash
# Round 2, session 2 measurement pass on one B200: GPU tests, smoke, ncu summaries of every
# config's traversal kernel (profile_r02.sh, read by bench.py), the bench line (cfg2 headline +
# per_config cfg1-5 + e2e) and the reference arm.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out/s2
O=gpurun_out/s2
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.used --format=csv > $O/gpu.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 1200 python -m pytest tests -q -m gpu > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 1800 bash scripts/profile_r02.sh > $O/profile.log 2>&1
cp profiles/r02/ncu_summary.json $O/ 2>/dev/null
timeout 1200 python bench.py > $O/bench_full.log 2>&1; echo "rc=$?" >> $O/bench_full.log
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > $O/bench_ref.log 2>&1; echo "rc=$?" >> $O/bench_ref.log
