python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -3
timeout 900 python -m pytest tests/test_gpu_multirank.py -q -x 2>&1 | grep -v "^  File" | tail -20
timeout 1500 python -m pytest tests -m gpu -q 2>&1 | grep -v "^  File" | tail -6
