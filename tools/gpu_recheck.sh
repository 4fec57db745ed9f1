# re-entry check: build, smoke, the GPU suite, one default bench line
set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -3
timeout 1500 python -m pytest tests -m gpu -q 2>&1 | grep -v "^  File" | tail -6
timeout 600 python bench.py > gpurun_out/bench_recheck.json 2> gpurun_out/bench_recheck.err; tail -2 gpurun_out/bench_recheck.err; cat gpurun_out/bench_recheck.json
