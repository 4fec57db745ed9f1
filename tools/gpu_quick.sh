set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -5
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -5
timeout 900 python bench.py --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench_q.json 2> gpurun_out/bench_q.err; tail -c 1500 gpurun_out/bench_q.json; tail -3 gpurun_out/bench_q.err
timeout 900 python tools/quick_run.py --config c2 --reps 2 2>&1 | tail -16
