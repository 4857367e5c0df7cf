cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
O=gpurun_out/ab_heavy2.log
run() { echo "$*" >> $O; env "$@" LUSYM_DEBUG_PLAN=1 timeout 300 python scripts/exp_ranges.py 3 0:1048576 >> $O 2>&1; }
run X=0
for x in 4096 16384 65536; do for t in 128 256; do run LUSYM_HEAVY_TOP=$x LUSYM_HEAVY_NT=$t; done; done
run X=0
