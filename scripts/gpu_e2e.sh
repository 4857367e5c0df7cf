cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out/e2e
timeout 600 python -m pytest tests/test_bound.py tests/test_gpu_parity.py -x -q -k "bound or run_host" > gpurun_out/e2e/t.log 2>&1; echo "rc=$?" >> gpurun_out/e2e/t.log
timeout 600 python bench.py --steps 5 --warmup 3 --per-config "" --no-numeric --e2e-steps 4 > gpurun_out/e2e/bench_cfg2.log 2>&1; echo "rc=$?" >> gpurun_out/e2e/bench_cfg2.log
timeout 600 python bench.py --steps 5 --warmup 3 --per-config "" --no-numeric --e2e-steps 4 --e2e-two-call --no-cpu-baseline > gpurun_out/e2e/bench_cfg2_two.log 2>&1; echo "rc=$?" >> gpurun_out/e2e/bench_cfg2_two.log
