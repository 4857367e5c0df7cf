cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
for r in 1 2 3 4; do for pad in 0 32 96; do echo "PAD=$pad" >> gpurun_out/pad.log; LUSYM_SLOT_PAD=$pad timeout 300 python scripts/exp_ranges.py 3 0:1048576 >> gpurun_out/pad.log 2>&1; done; done
