mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:eval_ -s 1 -c 1 -o gpurun_out/prof_eval_r2b -f python tools/prof_driver.py eval 2 > gpurun_out/ncu_eval_r2b.log 2>&1; tail -1 gpurun_out/ncu_eval_r2b.log
