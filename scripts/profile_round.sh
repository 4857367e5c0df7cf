#!/bin/bash
# Profiling pass for one round (run under gpurun, 1 GPU).  Writes raw reports to gpurun_out/;
# scripts/summarize_ncu.py turns them into profiles/<round>/ summaries.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
CFG=${CFG:-2}
# 1. every launch of one bench step with its device time (cold-cache, serialised)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_cfg${CFG}.csv \
    timeout 600 python bench.py --profile --config $CFG --steps 1 --warmup 1 > gpurun_out/launches_run.log 2>&1
# 2. full section set on the dominant kernel (the fill2 traversal, staged count pass), one launch
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fill2_kernel -s 1 -c 1 \
    -f -o gpurun_out/fill2_cfg${CFG} \
    timeout 600 python bench.py --profile --config $CFG --steps 1 --warmup 1 > gpurun_out/ncu_fill2.log 2>&1
# 3. the placement copy (emit) and the Kahn kernel
timeout 600 ncu --set full --clock-control none -k regex:"k_place|k_kahn|k_rank" -s 0 -c 3 \
    -f -o gpurun_out/aux_cfg${CFG} \
    timeout 600 python bench.py --profile --config $CFG --steps 1 --warmup 1 > gpurun_out/ncu_aux.log 2>&1
ls -la gpurun_out
