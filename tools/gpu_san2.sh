# compute-sanitizer on the current kernels (16-byte gather, zero-smem on-demand) + C4 timeline
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
rm -f gpurun_out/sanitize_summary.log
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_run.py > gpurun_out/sanitize_$tool.log 2>&1; echo "$tool rc=$?" >> gpurun_out/sanitize_summary.log
  tail -3 gpurun_out/sanitize_$tool.log >> gpurun_out/sanitize_summary.log
done
cat gpurun_out/sanitize_summary.log
ASCETIC_TRACE=2 timeout 900 python tools/quick_run.py --config c4 --reps 2 > gpurun_out/c4t_q.log 2> gpurun_out/c4t_trace.txt
grep -E "^\{'t'" gpurun_out/c4t_q.log | tail -6 | cut -c1-420
