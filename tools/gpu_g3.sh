python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 compute-sanitizer --tool memcheck --error-exitcode 9 python tools/sanitize_run.py 2>&1 | tail -2
timeout 900 compute-sanitizer --tool memcheck --error-exitcode 9 python -m pytest tests/test_gpu_parity.py -q -x -k "unaligned or tiny" 2>&1 | tail -2
for r in 1 2; do timeout 600 python tools/quick_run.py --config c2 --reps 3 --quiet 2>&1 | grep -E "kernels" | tail -1 | cut -c1-300; done
ASC_GATHER_OLD=1 timeout 600 python tools/quick_run.py --config c2 --reps 3 --quiet 2>&1 | grep -E "kernels" | tail -1 | cut -c1-300
