# compute-sanitizer evidence for the eval32 TMA/mbarrier ring, cp.async staging and K4/patch
# kernels: memcheck, racecheck, synccheck, initcheck on
# tests/tools/sanitize_run.py, with one and two candidates per lane.  Logs -> gpurun_out/san_*.log
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
python tests/tools/sanitize_run.py > gpurun_out/san_plain.log 2>&1; echo "rc=$?" >> gpurun_out/san_plain.log
for cpl in 1 2; do
  for tool in ${TOOLS:-memcheck racecheck synccheck initcheck}; do
    extra=""
    [ $tool = memcheck ] && extra="--leak-check no"
    [ $tool = racecheck ] && extra="--racecheck-report all"
    d4=1; [ $cpl = 2 ] && [ $tool = memcheck ] && d4=0
    SAN_D4=$d4 PESTO_EVAL32_CPL=$cpl timeout 1500 $CS --tool $tool $extra --print-limit 50 \
      python tests/tools/sanitize_run.py > gpurun_out/san_${tool}_cpl${cpl}.log 2>&1
    echo "rc=$?" >> gpurun_out/san_${tool}_cpl${cpl}.log
  done
done
echo done
