cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out/e2e
LUSYM_DEBUG_CREATE=1 timeout 600 python bench.py --steps 3 --warmup 3 --per-config "" --no-numeric --e2e-steps 3 --no-cpu-baseline > gpurun_out/e2e/bench_dbg.log 2> gpurun_out/e2e/bench_dbg.err; echo "rc=$?" >> gpurun_out/e2e/bench_dbg.log
LUSYM_DEBUG_CREATE=1 timeout 600 python scripts/e2e_probe.py --config 2 --steps 4 > gpurun_out/e2e/probe_dbg.log 2>&1
