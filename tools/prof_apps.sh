#!/bin/bash
# ncu --set full of each app's dominant kernel(s), per variant (one launch each,
# after the first steps); raw + details pages come back as CSV (the reports
# stay in /tmp on the box). Summarise here with tools/ncu_apps_summary.py.
#   APPS="ray nbody" VARIANTS="typeptr cuda" bash tools/prof_apps.sh
mkdir -p gpurun_out
cap() {  # name app variant kernel-regex [skip]
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "$4" \
      -s ${5:-1} -c 1 -o /tmp/$1 -f python tools/prof_app.py $2 --variant $3 --steps 3 > gpurun_out/$1.log 2>&1
  ncu -i /tmp/$1.ncu-rep --page raw --csv > gpurun_out/$1.raw.csv 2>/dev/null
  ncu -i /tmp/$1.ncu-rep --page details --csv > gpurun_out/$1.details.csv 2>/dev/null
}
kern() {  # app -> kernel regex of its dominant dispatch
  case $1 in
    ray) echo "regex:k_ray_(direct|virtual)";;
    gen) echo "regex:k_step_.*gen::";;
    gol) echo "regex:k_step_.*gol::";;
    traf) echo "regex:traf::App, \(int\)1";;
    stut) echo "regex:stut::App, \(int\)1";;
    nbody) echo "regex:nbody::App, \(int\)0";;
    collide) echo "regex:collide::App, \(int\)0";;
    graph-pr) echo "regex:graph::App, \(int\)4";;
    graph-cc) echo "regex:graph::App, \(int\)2";;
    graph-bfs) echo "regex:graph::App, \(int\)0";;
  esac
}
for a in ${APPS:-ray nbody gen gol traf stut collide graph-pr}; do
  for v in ${VARIANTS:-typeptr coal cuda}; do
    [ "$a" = gen ] && [ "$v" = cuda ] && v=cuda_packed  # 3 x 16.8M device `new`s take ~6 min
    cap prof_${a}_${v} $a $v "$(kern $a)"
  done
done
