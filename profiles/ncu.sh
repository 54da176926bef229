#!/bin/bash
# Profiling recipe used for profiles/ (run under gpurun on one B200; see B200_PROFILING.md).
# 1) launch list of the bench command's config-2 part (cold-cache, serialised: compare
#    shares, not absolutes)
# 2) one `ncu --set full` capture per dispatch variant of the config-2 kernel (T=4 random,
#    n=2^26); the raw page comes back as CSV (reports stay in /tmp on the box)
# 3) the per-app kernels: tools/prof_apps.sh
#   python tools/ncu_summary.py --tag r2 --n 67108864 gpurun_out/prof_*_T4.raw.csv \
#       --launches gpurun_out/launches.csv
set -x
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
B="python bench.py --steps 4 --warmup 3 --no-variants --no-e2e --no-cpu --apps="
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv $B --variant typeptr > $OUT/launches_bench.log 2>&1
for v in typeptr coal sharedoa; do
  case $v in sharedoa) K=regex:k_dispatch_virtual;; *) K="regex:k_dispatch_(grouped|sorted|pipe)";; esac
  ncu --set full --clock-control none --import-source on -k $K -s 3 -c 1 -o /tmp/prof_${v}_T4 -f \
      $B --variant $v --T ${T:-4} > $OUT/prof_${v}.log 2>&1
  ncu -i /tmp/prof_${v}_T4.ncu-rep --page raw --csv > $OUT/prof_${v}_T4.raw.csv 2>/dev/null
done
