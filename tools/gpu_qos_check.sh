mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_qos.py -q -x -p no:cacheprovider 2>&1 | tail -2
timeout 900 python tools/elastic_sweep.py > gpurun_out/r02_elastic_sweep.json 2> gpurun_out/elastic_sweep.err; tail -c 200 gpurun_out/r02_elastic_sweep.json
