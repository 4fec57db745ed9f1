python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_run.py > gpurun_out/sanitize_$tool.log 2>&1; echo "$tool rc=$?" >> gpurun_out/sanitize_summary.log
  tail -3 gpurun_out/sanitize_$tool.log >> gpurun_out/sanitize_summary.log
done
timeout 1500 python tools/quick_run.py --config c4 --reps 2 --quiet --oracle > gpurun_out/c4.log 2>&1
