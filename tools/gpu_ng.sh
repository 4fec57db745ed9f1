#!/bin/bash
# A/B of the gather's loads-per-lane-per-round (ASC_GATHER_NG) on the C2 bench, interleaved.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/ng_build.log 2>&1
for rep in 1 2; do for ng in 4 5 6 8; do
  ASC_GATHER_NG=$ng timeout 300 python bench.py --no-cpu-baseline --e2e-steps 0 --steps 5 --warmup 3 > gpurun_out/ng_${ng}_${rep}.json 2> gpurun_out/ng_${ng}_${rep}.err
  python -c "
import json;d=json.load(open('gpurun_out/ng_${ng}_${rep}.json'));r=d['roofline']['per_kernel']['gather']
print('NG=$ng rep=$rep', round(d['value'],3),'GTEPS', round(r['achieved'],2),'GB/s gather', round(d['ms_per_step'],2),'ms')" >> gpurun_out/ng_ab.log 2>&1
done; done
cat gpurun_out/ng_ab.log
