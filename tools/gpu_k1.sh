#!/bin/bash
# K1 variants on one box: eval parity tests (default and K1_TEST_VARIANT), then C5 timings per SPLIT_EVAL_VARIANT.
mkdir -p gpurun_out
for tv in -1 ${K1_TEST_VARIANT:-}; do
  SPLIT_EVAL_VARIANT=$tv timeout 900 python -m pytest tests/test_gpu_eval.py -q -x --timeout 300 -p no:cacheprovider > gpurun_out/pytest_eval_$tv.log 2>&1; echo "variant $tv: $(tail -1 gpurun_out/pytest_eval_$tv.log)"
done
for v in ${K1_VARIANTS:--1}; do
  SPLIT_EVAL_VARIANT=$v timeout 120 python tools/eval_sweep.py c5 2>&1 | tail -1 | sed "s/^/v=$v /"
done > gpurun_out/eval_ab.log 2>&1; cat gpurun_out/eval_ab.log
