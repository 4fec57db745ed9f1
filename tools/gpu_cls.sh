python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
timeout 600 python tools/quick_run.py --config c2 --reps 3 --quiet 2>&1 | grep -E "kernels" | tail -1 | cut -c1-260
timeout 600 python tools/quick_run.py --config c4 --scale-override 26 --reps 2 --quiet 2>&1 | grep -E "kernels" | tail -1 | cut -c1-260
