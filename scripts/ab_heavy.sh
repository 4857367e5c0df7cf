# cfg3: the last rows in a shared-map class next to the sparse class (LUSYM_HEAVY_TOP rows,
# LUSYM_HEAVY_GRID rows in flight), count pass of all rows
cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
O=gpurun_out/ab_heavy.log
run() { echo "$*" >> $O; env "$@" LUSYM_DEBUG_PLAN=1 timeout 300 python scripts/exp_ranges.py 3 0:1048576 >> $O 2>&1; }
run LUSYM_HEAVY_TOP=0
for x in 2048 4096 16384; do for g in 0 74; do run LUSYM_HEAVY_TOP=$x LUSYM_HEAVY_GRID=$g; done; done
run LUSYM_HEAVY_TOP=0
