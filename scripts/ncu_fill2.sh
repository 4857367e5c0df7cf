#!/bin/bash
# ncu --set full of the first fill2 launch (the top row class) for each config in CFGS (under gpurun)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for c in ${CFGS:-2}; do
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:fill2_kernel -s ${SKIP:-1} -c 1 \
      -f -o gpurun_out/fill2_cfg${c} \
      timeout 900 python bench.py --profile --config $c --steps 1 --warmup 1 > gpurun_out/ncu_fill2_cfg$c.log 2>&1
  echo "cfg$c rc=$?"
done
ls -la gpurun_out
