#!/bin/bash
# One GPU round (run on the GPU box via gpurun): tests, smoke, bench line, launch list, full ncu captures
# (kept on the box under /tmp/ncu; their summaries and CSV exports go to gpurun_out/).  ROUND_TESTS=0 skips tests.
set -u
mkdir -p gpurun_out /tmp/ncu
TAG=${TAG:-r02}
if [ "${ROUND_TESTS:-1}" = 1 ]; then
  timeout 1800 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
  timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
fi
timeout 900 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; tail -c 300 gpurun_out/bench_full.json; echo
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-ga-big --no-qos --no-c3 --no-c4 > gpurun_out/launch_bench.log 2>&1
N=/tmp/ncu
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ga_kernel -s 1 -c 1 -o $N/prof_ga -f python tools/prof_driver.py ga 2 500 > gpurun_out/ncu_ga.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval_ -s 1 -c 1 -o $N/prof_eval -f python tools/prof_driver.py eval 2 > gpurun_out/ncu_eval.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ga_kernel -s 1 -c 1 -o $N/prof_ga_1m -f python tools/prof_driver.py ga_1m 1 20 > gpurun_out/ncu_ga_1m.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ga_kernel -s 1 -c 1 -o $N/prof_ga_4m -f python tools/prof_driver.py ga_big 1 20 > gpurun_out/ncu_ga_4m.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:qos_kernel -s 1 -c 1 -o $N/prof_qos -f python tools/prof_driver.py qos 2 > gpurun_out/ncu_qos.log 2>&1
SPLIT_NCU_DIR=$N SPLIT_PROF_OUT=gpurun_out python tools/summarize_profiles.py $TAG > /dev/null 2>&1
for r in prof_eval prof_ga prof_ga_1m; do
  ncu -i $N/$r.ncu-rep --page raw --csv > gpurun_out/${TAG}_${r}_raw.csv 2>/dev/null
  ncu -i $N/$r.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/${TAG}_${r}_source.csv 2>/dev/null
done
cp $N/prof_eval.ncu-rep gpurun_out/${TAG}_prof_eval.ncu-rep
du -sh gpurun_out; ls gpurun_out | tail -30
