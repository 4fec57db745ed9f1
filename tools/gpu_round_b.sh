# round-1 session B: full GPU tests, sanitizers on the new paths, ncu of the new kernels, PRD workloads
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -7
timeout 1200 python -m pytest tests -m gpu -q 2>&1 | grep -v "^  File" | tail -8
for tool in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_run.py > gpurun_out/sanitize_$tool.log 2>&1; echo "$tool rc=$?"
  grep -E "ERROR SUMMARY|mismatches" gpurun_out/sanitize_$tool.log | tail -2
done
for k in "k_chunk_access" "k_copy_chunks" "k_static_rebits" "k_static_med<1, true>" "k_ondemand<4>" "k_static_med<4, false>" "k_finalize_prd"; do
  f=$(echo "$k" | tr -dc 'a-z0-9_')
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:$k" -s 5 -c 1 \
      -o gpurun_out/prof_$f -f python tools/ncu_new_kernels.py > gpurun_out/ncu_$f.log 2>&1
  echo "ncu $k rc=$?"
done
ABLATION_ONLY=prd timeout 1800 python tools/ablation.py c1 c3 c4 2>&1 | grep -v "^{" | tail -12
cp gpurun_out/ablation.md gpurun_out/ablation_prd.md
ls gpurun_out
