# timelines of the current build: C3 (PR, 6 iterations) and C4 (CC), ASCETIC_TRACE spans
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
ASCETIC_TRACE=1 timeout 900 python tools/quick_run.py --config c3 --iters 6 --reps 2 --quiet > gpurun_out/c3_q.log 2> gpurun_out/c3_trace.txt
tail -4 gpurun_out/c3_q.log
ASCETIC_TRACE=1 timeout 900 python tools/quick_run.py --config c4 --reps 2 > gpurun_out/c4_q.log 2> gpurun_out/c4_trace.txt
tail -12 gpurun_out/c4_q.log
