# zero-shared-memory on-demand kernel (ASC_OND_GLOBAL=1) vs the smem-staged one
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
ASC_OND_GLOBAL=1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_prd.py -q -x 2>&1 | tail -2
for v in "ASC_OND_GLOBAL=0" "ASC_OND_GLOBAL=1"; do
  echo "== c3 6 it [$v]"
  env $v ASCETIC_TRACE=2 timeout 900 python tools/quick_run.py --config c3 --iters 6 --reps 2 --quiet 2> gpurun_out/c3g_$v.txt | grep -E "kernels" | cut -c1-330
  echo "== c2 [$v]"; env $v timeout 600 python tools/quick_run.py --config c2 --reps 3 --quiet 2>&1 | grep -E "kernels" | tail -1 | cut -c1-300
  echo "== c4/26 [$v]"; env $v timeout 600 python tools/quick_run.py --config c4 --scale-override 26 --reps 2 --quiet 2>&1 | grep -E "kernels" | tail -1 | cut -c1-300
done
