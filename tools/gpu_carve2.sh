# static-kernel carveout sweep (percent of max shared); other kernels default
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
for v in "ASC_CARVE_STATIC=-1" "ASC_CARVE_STATIC=25" "ASC_CARVE_STATIC=40" "ASC_CARVE_STATIC=60"; do
  echo "== c3 6 it [$v]"
  env $v ASCETIC_TRACE=2 timeout 900 python tools/quick_run.py --config c3 --iters 6 --reps 2 --quiet 2> gpurun_out/c3d_$v.txt | grep -E "kernels" | cut -c1-330
  echo "== c2 [$v]"; env $v timeout 600 python tools/quick_run.py --config c2 --reps 3 --quiet 2>&1 | grep -E "kernels" | tail -1 | cut -c1-300
done
