cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
: > gpurun_out/quick.log
for w in 0 600 1200 2400; do
    r=$(PESTO_ND_MAX_WARPS=$w timeout 300 python scripts/time_nondelay.py inception_v3_2dev 8192 2>&1 | tail -1)
    echo "maxwarps=$w $r" >> gpurun_out/quick.log
done
