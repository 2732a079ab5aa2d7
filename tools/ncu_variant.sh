mkdir -p gpurun_out
SPLIT_EVAL_VARIANT=10 timeout 600 ncu --set full --clock-control none --import-source on -k regex:eval_batch -s 1 -c 1 -o gpurun_out/prof_eval_v10 python tools/prof_driver.py eval 2 > gpurun_out/ncu_eval10.log 2>&1
tail -3 gpurun_out/ncu_eval10.log
