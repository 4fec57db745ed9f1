python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_replace.py tests/test_gpu_prd.py -q -x 2>&1 | tail -2
for a in bfs sssp cc pr; do
  echo "== resident $a (RMAT-24, budget 1.2x CSR)"
  it=0; [ $a = pr ] && it=10
  timeout 600 python tools/quick_run.py --config c2 --algo-override $a --budget-mult 1.2 --reps 2 --quiet --iters $it --static-ctas 4,8 2>&1 | grep -E "static_ctas|GTEPS" | cut -c1-60,200-400
done
