#!/bin/bash
# ncu --set full of the collision update and N-body update kernels (one launch each);
# reports stay in /tmp on the box, their raw + details pages come back as CSV.
mkdir -p gpurun_out
cap() {  # name app variant kernel-regex
  ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "$4" -s 1 -c 1 \
      -o /tmp/$1 -f python tools/prof_app.py $2 --variant $3 --steps 2 > gpurun_out/$1.log 2>&1
  ncu -i /tmp/$1.ncu-rep --page raw --csv > gpurun_out/$1.raw.csv 2>/dev/null
  ncu -i /tmp/$1.ncu-rep --page details --csv > gpurun_out/$1.details.csv 2>/dev/null
  ncu -i /tmp/$1.ncu-rep --page source --csv --print-source sass > /tmp/$1.src.csv 2>/dev/null
  head -c 8000000 /tmp/$1.src.csv > gpurun_out/$1.src.csv
}
for a in ${APPS:-collide nbody}; do
  for v in ${VARIANTS:-typeptr cuda}; do
    cap prof_${a}_${v} $a $v "regex:${a}::App, \(int\)0"
  done
done
