python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
bash tools/gpu_resident.sh 2>&1 | grep -E "==|kernels" | awk 'NR%3!=2'
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench_q.json 2> gpurun_out/bench_q.err; python -c "
import json; d=json.loads(open('gpurun_out/bench_q.json').read().strip().splitlines()[-1]); print('value',d['value'],'ms',d['ms_per_step'],'e2e',d['e2e']['value'],d['e2e']['ms_per_step']); print(d['link']); print({k:(v['time_s'],v['achieved']) for k,v in d['roofline']['per_kernel'].items()})"
