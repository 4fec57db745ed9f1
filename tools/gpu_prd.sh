python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_prd.py -x -q 2>&1 | grep -v "^  File" | tail -25
timeout 1200 python -m pytest tests -m gpu -q 2>&1 | grep -v "^  File" | tail -8
