# A/B of the static-hit kernel batching factors (dev builds under _ab/, not rebuilt here)
for a in bfs sssp cc pr; do
  it=0; [ $a = pr ] && it=10
  for v in old v11 v21 v22 v42; do
    echo "== $v resident $a"
    (cd _ab/$v && timeout 600 python tools/quick_run.py --config c2 --algo-override $a --budget-mult 1.2 --reps 2 --quiet --iters $it --static-ctas 4,8 2>&1 | grep -E "kernels" | cut -c1-48)
  done
done
