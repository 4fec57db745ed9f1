python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
rm -f gpurun_out/sanitize_summary.log
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_run.py > gpurun_out/sanitize_$tool.log 2>&1; echo "$tool rc=$?" >> gpurun_out/sanitize_summary.log
  tail -3 gpurun_out/sanitize_$tool.log >> gpurun_out/sanitize_summary.log
done
cat gpurun_out/sanitize_summary.log
timeout 900 compute-sanitizer --tool memcheck --error-exitcode 9 python -m pytest tests/test_gpu_parity.py -q -x -k "unaligned or tiny" 2>&1 | tail -3
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
timeout 600 python tools/quick_run.py --config c2 --reps 3 --quiet 2>&1 | grep -E "kernels" | tail -1 | cut -c1-300
