# gather / on-demand co-scheduling experiment (C4-shaped at scale 26, C2): dev knobs via env
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
for v in "" "ASC_GATHER_DSMEM=100000" "ASC_OND_CTAS=740" "ASC_OND_CTAS=444" "ASC_GATHER_DSMEM=100000 ASC_OND_CTAS=740"; do
  echo "== c4/26 [$v]"
  env $v timeout 600 python tools/quick_run.py --config c4 --scale-override 26 --reps 2 --quiet 2>&1 | grep -E "^buffers|kernels" | tail -2 | cut -c1-400
done
for v in "" "ASC_GATHER_DSMEM=100000" "ASC_OND_CTAS=740"; do
  echo "== c2 [$v]"
  env $v timeout 600 python tools/quick_run.py --config c2 --reps 3 --quiet 2>&1 | grep -E "^buffers|kernels" | tail -2 | cut -c1-400
done
