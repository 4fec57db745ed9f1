# new 16-byte cover gather: parity suites, then A/B against the 4/8-byte gather on C2 and C4-shaped
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | grep -v "^  File" | tail -8
for v in "ASC_GATHER_OLD=1" "ASC_GATHER_OLD=0"; do
  echo "== c2 [$v]"; env $v timeout 600 python tools/quick_run.py --config c2 --reps 3 --quiet 2>&1 | grep -E "kernels" | tail -1 | cut -c1-300
  echo "== c4/26 [$v]"; env $v timeout 600 python tools/quick_run.py --config c4 --scale-override 26 --reps 2 --quiet 2>&1 | grep -E "kernels" | tail -1 | cut -c1-300
done
