# ncu --set full of one k_integrate launch (step 2 of config 2) for integrator variant $V
V=${V:-0}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_integrate -s 2 -c 1 -o gpurun_out/prof_v$V -f python tools/ab_eval.py 2 3 $V > gpurun_out/ncu_v$V.log 2>&1
tail -2 gpurun_out/ncu_v$V.log
