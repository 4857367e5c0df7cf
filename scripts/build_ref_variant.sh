#!/bin/bash
# Build lib/variants/liblusym_<name>.so from the CUDA sources of git revision REV (default HEAD),
# for A/B runs of the working tree against a committed kernel (scripts/ab_variants.sh).
set -e
cd "$(dirname "$0")/.."
REV=${1:-HEAD}; NAME=${2:-head}
T=$(mktemp -d)
git archive "$REV" paper_conf_ppopp_xia0ar23_b200/csrc include | tar -x -C "$T"
mkdir -p paper_conf_ppopp_xia0ar23_b200/lib/variants "$T/obj"
for f in "$T"/paper_conf_ppopp_xia0ar23_b200/csrc/*.cu; do
  nvcc -c "$f" -o "$T/obj/$(basename "$f").o" -O3 -lineinfo -std=c++17 -Xcompiler -fPIC \
      -gencode arch=compute_100a,code=sm_100a -I "$T/include" &
done
wait
nvcc -shared -o paper_conf_ppopp_xia0ar23_b200/lib/variants/liblusym_$NAME.so "$T"/obj/*.o \
    -gencode arch=compute_100a,code=sm_100a
rm -rf "$T"
echo built paper_conf_ppopp_xia0ar23_b200/lib/variants/liblusym_$NAME.so
