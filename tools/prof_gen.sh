# per-kernel launch list (ncu gpu__time_duration) of the first GEN / GOL generations per variant
mkdir -p gpurun_out
for v in sharedoa coal typeptr; do
  timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
     --log-file gpurun_out/launch_gen_$v.csv python tools/prof_app.py gen --variant $v --steps 4 > /dev/null 2>&1
  timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
     --log-file gpurun_out/launch_gol_$v.csv python tools/prof_app.py gol --variant $v --steps 4 > /dev/null 2>&1
done
timeout 300 python tools/sweep_apps.py --apps golgraph --out gpurun_out/sweep_golgraph > gpurun_out/sweep_golgraph.log 2>&1
