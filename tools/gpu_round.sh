#!/bin/bash
# One GPU round: tests, bench line, launch list, full ncu captures (run on the GPU box via gpurun).
set -u
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; tail -c 400 gpurun_out/bench_full.json; echo
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-ga-big --no-qos --no-c3 --no-c4 > gpurun_out/launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ga_kernel -s 1 -c 1 -o gpurun_out/prof_ga python tools/prof_driver.py ga 2 500 > gpurun_out/ncu_ga.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval_batch -s 1 -c 1 -o gpurun_out/prof_eval python tools/prof_driver.py eval 2 > gpurun_out/ncu_eval.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:qos_kernel -s 1 -c 1 -o gpurun_out/prof_qos python tools/prof_driver.py qos 2 > gpurun_out/ncu_qos.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:qos_kernel -s 1 -c 1 -o gpurun_out/prof_qos_el python tools/prof_driver.py qos_el 2 > gpurun_out/ncu_qos_el.log 2>&1
ls -la gpurun_out | tail -14
