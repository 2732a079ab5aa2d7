#!/bin/bash
# K1 A/B on one GPU box (via gpurun): parity tests, variant timings, ncu of the default K1.
set -u
mkdir -p gpurun_out
export PYTHONDONTWRITEBYTECODE=1
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; tail -5 gpurun_out/pytest_gpu.log
for v in ${K1_VARIANTS:--1 100 101 102 103 104}; do
  SPLIT_EVAL_VARIANT=$v timeout 300 python tools/eval_sweep.py c5 2>&1 | sed "s/^/v=$v /"
done > gpurun_out/eval_ab.log 2>&1; cat gpurun_out/eval_ab.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:eval_ -s 1 -c 1 -o gpurun_out/prof_eval_r2 -f python tools/prof_driver.py eval 2 > gpurun_out/ncu_eval_r2.log 2>&1; tail -2 gpurun_out/ncu_eval_r2.log
timeout 600 python tools/island_probe.py > gpurun_out/island_probe.log 2>&1; cat gpurun_out/island_probe.log
