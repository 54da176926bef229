# ncu --set full of the GraphChi-vEN kernels (one launch each): the vertex
# gather with nested edge calls and the per-edge pull, TypePointer and SharedOA
mkdir -p gpurun_out
for v in typeptr sharedoa; do
  case $v in sharedoa) K=k_dispatch_virtual;; *) K=k_dispatch_sorted;; esac
  for name in pr-gather pr-pull; do
    case $name in pr-gather) P="VtxApp, \(int\)3";; *) P="EdgeApp, \(int\)0";; esac
    timeout 400 ncu --set full --import-source on --clock-control none --kernel-name-base demangled \
      -k "regex:${K}<vf::graph_en::${P}" -s 1 -c 1 -o /tmp/prof_en_${name}_${v} -f \
      python tools/prof_app.py graph-en-pr --variant $v --scale ${SCALE:-24} > gpurun_out/prof_en_${name}_${v}.log 2>&1
    ncu -i /tmp/prof_en_${name}_${v}.ncu-rep --page raw --csv > gpurun_out/prof_en_${name}_${v}.raw.csv 2>/dev/null
    ncu -i /tmp/prof_en_${name}_${v}.ncu-rep --page details > gpurun_out/prof_en_${name}_${v}.details.txt 2>/dev/null
  done
done
