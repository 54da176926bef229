# ncu --set full of the graph dispatch kernels (one launch each); the box keeps
# only CSV/text exports (reports are too large to bring back), see profiles/
mkdir -p gpurun_out
for m in "graph-pr:4" "graph-cc:2" "graph-bfs:0"; do
  app=${m%%:*}; k=${m#*:}
  timeout 300 ncu --set full --import-source on --clock-control none --kernel-name-base demangled \
    -k "regex:k_dispatch_sorted<vf::graph::App, \(int\)$k," -s 1 -c 1 -o /tmp/prof_${app} -f \
    python tools/prof_app.py $app > gpurun_out/prof_${app}.log 2>&1
  ncu -i /tmp/prof_${app}.ncu-rep --page raw --csv > gpurun_out/prof_${app}.raw.csv 2>/dev/null
  ncu -i /tmp/prof_${app}.ncu-rep --page details > gpurun_out/prof_${app}.details.txt 2>/dev/null
  ncu -i /tmp/prof_${app}.ncu-rep --page source --csv > gpurun_out/prof_${app}.source.csv 2>/dev/null
done
