mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_ga.py -q -x --timeout 600 -p no:cacheprovider > gpurun_out/pytest_ga.log 2>&1; tail -15 gpurun_out/pytest_ga.log
timeout 600 python tools/island_probe.py > gpurun_out/island_probe.log 2>&1; cat gpurun_out/island_probe.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/island_launches.csv python tools/island_probe.py 8 10 > /dev/null 2>&1; python tools/ncu_launches.py gpurun_out/island_launches.csv 12
bash tools/gpu_synctrace.sh
