cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
for r in 1 2; do for g in 4 8 16; do for hd in 2 4; do echo "G=$g HEAD=$hd" >> gpurun_out/mcl.log; LUSYM_MERGE_CLUSTER=$g LUSYM_MERGE_GRID_HEAD=$hd timeout 300 python scripts/merge_stats.py >> gpurun_out/mcl.log 2>&1; done; done; done
