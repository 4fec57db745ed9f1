for a in bfs sssp cc pr; do
  echo "== resident $a (RMAT-24, budget 1.2x CSR)"
  it=0; [ $a = pr ] && it=10
  timeout 600 python tools/quick_run.py --config c2 --algo-override $a --budget-mult 1.2 --reps 2 --quiet --iters $it 2>&1 | grep -v "^gen\|^load" | tail -3
done
