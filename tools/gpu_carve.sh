# A/B of the uniform shared-memory carveout (ASC_NO_CARVE=1 = per-kernel default)
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
for v in "ASC_NO_CARVE=1" "ASC_NO_CARVE=0"; do
  echo "== c3 6 it [$v]"
  env $v ASCETIC_TRACE=2 timeout 900 python tools/quick_run.py --config c3 --iters 6 --reps 2 --quiet 2> gpurun_out/c3c_$v.txt | grep -E "kernels|^buffers" | cut -c1-330
  echo "== c2 [$v]"; env $v timeout 600 python tools/quick_run.py --config c2 --reps 3 --quiet 2>&1 | grep -E "kernels" | tail -1 | cut -c1-300
  echo "== c4/26 [$v]"; env $v timeout 600 python tools/quick_run.py --config c4 --scale-override 26 --reps 2 --quiet 2>&1 | grep -E "kernels" | tail -1 | cut -c1-300
done
