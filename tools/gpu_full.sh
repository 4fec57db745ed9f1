set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -5
timeout 1500 python -m pytest tests -m gpu -x -q --durations=5 2>&1 | tail -12
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench_q.json 2> gpurun_out/bench_q.err; tail -c 1800 gpurun_out/bench_q.json; tail -3 gpurun_out/bench_q.err
