# tuning round: GPU parity, eval variants, bench, GA phase trace (run via gpurun)
set -u
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x --timeout 600 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; tail -5 gpurun_out/pytest_gpu.log
for v in ${EVAL_VARIANTS:-}; do echo "variant $v"; SPLIT_EVAL_VARIANT=$v timeout 120 python tools/eval_sweep.py c5; done
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench_exp.json 2> gpurun_out/bench_exp.err; tail -3 gpurun_out/bench_exp.err; python -c "
import json;d=json.loads(open('gpurun_out/bench_exp.json').read().strip().splitlines()[-1])
print('GA',d['value'],d['ms_per_step'],'e2e',d['e2e']['value'],'eval',d['eval_batch']['evals_per_s'])
for k in ('ga_hbm_regime','qos_sim','exact'): print(k, json.dumps(d.get(k))[:900])"
if [ -n "${TRACE:-}" ]; then
SPLIT_TRACE_BUILD=1 python -m paper_conf_icpp_luoyww0023_b200.build --force > /dev/null 2>&1; SPLIT_TRACE=gpurun_out/trace.csv python tools/trace_ga.py run; python tools/trace_ga.py show gpurun_out/trace.csv
fi
