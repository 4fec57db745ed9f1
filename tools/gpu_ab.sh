# A/B: resident static-hit kernels, old (_ab/old, before batching) vs current, same box
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
(cd _ab/old && python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1)
for a in bfs sssp cc pr; do
  it=0; [ $a = pr ] && it=10
  for v in old new; do
    d=.; [ $v = old ] && d=_ab/old
    echo "== $v resident $a"
    (cd $d && timeout 600 python tools/quick_run.py --config c2 --algo-override $a --budget-mult 1.2 --reps 2 --quiet --iters $it --static-ctas 4,8 2>&1 | grep -E "kernels" | cut -c1-70)
  done
done
