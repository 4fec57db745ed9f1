# resident PR static pull: contrib in L2 (RMAT-24, 67 MB) vs beyond L2 (friendster-shaped, 262 MB)
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python tools/quick_run.py --config c2 --algo-override pr --budget-mult 1.2 --iters 5 --reps 2 --quiet 2>&1 | grep -E "kernels" | cut -c1-250
timeout 900 python tools/quick_run.py --config c3 --budget-mult 1.2 --iters 5 --reps 2 --quiet 2>&1 | grep -E "kernels" | cut -c1-250
