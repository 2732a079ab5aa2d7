mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_ga.py -q -x -p no:cacheprovider 2>&1 | tail -1
python tools/ga_c2_probe.py | tail -1
python tools/island_probe.py 2>&1 | grep -v NCCL
