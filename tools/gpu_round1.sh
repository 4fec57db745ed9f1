set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -20
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -30
timeout 600 python tools/quick_run.py --algo sssp --scale 20 --oracle 2>&1 | tail -30
timeout 600 python tools/quick_run.py --algo sssp --scale 20 --xfer 2 2>&1 | tail -5
timeout 600 python tools/quick_run.py --algo pr --scale 20 --iters 10 --oracle 2>&1 | tail -20
