# class boundaries at the largest shared map that adds rows in flight (LUSYM_TIGHT_CLASSES)
cd ${GRAFT_REPO_ROOT:-/root/repo}
mkdir -p gpurun_out
O=gpurun_out/ab_tight.log
run() { echo "$*" >> $O; env "$@" LUSYM_DEBUG_PLAN=1 timeout 600 python scripts/exp_ranges.py $C >> $O 2>&1; }
C="4 0:1048576"; run X=0; run LUSYM_TIGHT_CLASSES=1; run X=0; run LUSYM_TIGHT_CLASSES=1
C="5 0:262144"; run X=0; run LUSYM_TIGHT_CLASSES=1
C="2 0:64000"; run X=0; run LUSYM_TIGHT_CLASSES=1
C="3 0:1048576"; run X=0; run LUSYM_TIGHT_CLASSES=1
