python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
ASCETIC_TRACE=2 timeout 900 python tools/quick_run.py --config c3 --iters 4 --reps 1 --quiet > gpurun_out/c3s_q.log 2> gpurun_out/c3s_trace.txt
tail -2 gpurun_out/c3s_q.log | cut -c1-300
bash tools/gpu_profile.sh > /dev/null 2>&1
timeout 600 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err; cat gpurun_out/bench_c2.json | cut -c1-600
ls gpurun_out
