mkdir -p gpurun_out
SPLIT_TRACE_BUILD=1 python -m paper_conf_icpp_luoyww0023_b200.build --force > /dev/null 2>&1
SPLIT_TRACE=gpurun_out/sync_trace.csv timeout 300 python tools/island_probe.py 8 10
python tools/sync_trace.py gpurun_out/sync_trace.csv
