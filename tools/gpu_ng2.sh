#!/bin/bash
# sparse-exchange GPU tests again + gather CTAs sweep below the default at NG = 6 (C2)
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_multirank.py tests/test_gpu_nccl.py -q -k "sparse" 2>&1 | tail -2
timeout 900 python tools/quick_run.py --config c2 --reps 1 --quiet --sweep --sweep-ctas 32,48,64,96,64,48 --sweep-caps 0 2>&1 | grep gather_ctas
