# build + the GPU test suite (replacement tests first); used through gpurun
set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -6
timeout 900 python -m pytest tests/test_gpu_replace.py -x -q 2>&1 | tail -30
timeout 1200 python -m pytest tests -m gpu -q 2>&1 | tail -8
