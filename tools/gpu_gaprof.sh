mkdir -p gpurun_out
python tools/ga_big_probe.py 2>&1 | tail -4
# RUN launch of the 1M and 4M islands (20 generations each; -s 1: skip the INIT launch)
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ga_kernel -s 1 -c 1 -o gpurun_out/prof_ga_1m -f python tools/prof_driver.py ga_1m 1 20 > gpurun_out/ncu_ga_1m.log 2>&1; tail -1 gpurun_out/ncu_ga_1m.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ga_kernel -s 1 -c 1 -o gpurun_out/prof_ga_4m -f python tools/prof_driver.py ga_big 1 20 > gpurun_out/ncu_ga_4m.log 2>&1; tail -1 gpurun_out/ncu_ga_4m.log
