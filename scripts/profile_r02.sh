#!/bin/bash
# Round-2 profiles (under gpurun, one GPU): the traversal kernel of every config with
# `ncu --set full` (cfg4/cfg5 on their heaviest rows), the row-merge tail on cfg3,
# and the launch list of one cfg2 bench step.  Summarise here with scripts/summarize_ncu_r02.py.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out /tmp/prof
P=/tmp/prof
N="ncu --set full --import-source on --clock-control none -k fill2_kernel"
timeout 300 $N --launch-count 1 -o $P/p2_cfg1 python scripts/prof_count.py 1 > gpurun_out/p2_cfg1.log 2>&1
timeout 300 $N --launch-count 1 -o $P/p2_cfg2 python scripts/prof_count.py 2 > gpurun_out/p2_cfg2.log 2>&1
timeout 600 $N --launch-skip 1 --launch-count 1 -o $P/p2_cfg3 python scripts/prof_count.py 3 > gpurun_out/p2_cfg3.log 2>&1
timeout 600 $N --launch-skip 1 --launch-count 1 -o $P/p2_cfg4 python scripts/prof_count.py 4 1040000 0 > gpurun_out/p2_cfg4.log 2>&1
timeout 600 $N --launch-skip 1 --launch-count 1 -o $P/p2_cfg5 python scripts/prof_count.py 5 250000 0 > gpurun_out/p2_cfg5.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k k_merge_rows --launch-count 1 -o $P/p2_merge_cfg3 python scripts/prof_count.py 3 > gpurun_out/p2_merge.log 2>&1
# second runs without ncu: the rows' SV (the ncu run's own log has it too)
for c in "4 1040000 0" "5 250000 0"; do python scripts/prof_count.py $c >> gpurun_out/p2_nocu.log 2>&1; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_cfg2.csv python bench.py --profile --steps 1 --warmup 1 --per-config "" --no-e2e --no-cpu-baseline --no-numeric --no-verify > gpurun_out/p2_launches.log 2>&1

# summaries here on the box (the reports themselves are too large to bring back)
python scripts/summarize_ncu_r02.py cfg1=$P/p2_cfg1.ncu-rep:gpurun_out/p2_cfg1.log cfg2=$P/p2_cfg2.ncu-rep:gpurun_out/p2_cfg2.log cfg3=$P/p2_cfg3.ncu-rep:gpurun_out/p2_cfg3.log cfg4=$P/p2_cfg4.ncu-rep:gpurun_out/p2_cfg4.log cfg5=$P/p2_cfg5.ncu-rep:gpurun_out/p2_cfg5.log cfg3/k_merge_rows=$P/p2_merge_cfg3.ncu-rep > gpurun_out/p2_summary.log 2>&1
mkdir -p gpurun_out/r02prof
cp profiles/r02/ncu_summary.json profiles/r02/ncu_cfg*.txt gpurun_out/r02prof/ 2>/dev/null
for c in cfg1 cfg2 cfg3 cfg4 cfg5 merge_cfg3; do
  python scripts/ncu_hot.py $P/p2_$c.ncu-rep 3000 > gpurun_out/r02prof/hot_$c.txt 2>&1
  python scripts/ncu_regions.py $P/p2_$c.ncu-rep > gpurun_out/r02prof/regions_$c.txt 2>&1
  python scripts/ncu_funcs.py $P/p2_$c.ncu-rep > gpurun_out/r02prof/funcs_$c.txt 2>&1
  ncu -i $P/p2_$c.ncu-rep --page details --csv > gpurun_out/r02prof/details_$c.csv 2>/dev/null
done
python scripts/summarize_ncu.py r02 2 > gpurun_out/r02prof/launches_summary.txt 2>&1 || true
cp profiles/r02/launches_cfg2.txt gpurun_out/r02prof/ 2>/dev/null
