# the grid-wide tail (k_merge_grid) for short deferred-row lists vs the 4-CTA clusters
cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "deferred or cfg3_full or knobs" > gpurun_out/t_mgrid.log 2>&1; echo "rc=$?" >> gpurun_out/t_mgrid.log
O=gpurun_out/ab_mgrid.log
for v in 0 64 0 64; do echo "LUSYM_MERGE_GRID_MAX=$v" >> $O; LUSYM_MERGE_GRID_MAX=$v timeout 600 python bench.py --config 3 --steps 5 --warmup 3 --per-config "" --no-numeric --no-e2e --no-cpu-baseline > gpurun_out/b_mgrid_$v.log 2>&1; python -c "
import json; l=[x for x in open('gpurun_out/b_mgrid_$v.log') if x.startswith('{')][-1]; d=json.loads(l); print(d['ms_per_step'], d['phases_ms'], d['parity'][:60])" >> $O 2>&1; done
