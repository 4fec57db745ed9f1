# session C: batched static kernels — parity, resident throughput, ncu of the static kernels
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -6
timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | grep -v "^  File" | tail -8
bash tools/gpu_resident.sh 2>&1
for k in "k_static_med<\(int\)1, \(bool\)0>" "k_static_small<\(int\)1, \(bool\)0>" "k_static_med<\(int\)1, \(bool\)1>" "k_ondemand<\(int\)4>" "k_static_med<\(int\)4, \(bool\)0>"; do
  f=$(echo "$k" | tr -dc 'a-z0-9_')
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:$k" -s 3 -c 1 \
      -o gpurun_out/prof_$f -f python tools/ncu_new_kernels.py > gpurun_out/ncu_$f.log 2>&1
  echo "ncu $k rc=$?"
done
timeout 900 python bench.py --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench_c.json 2> gpurun_out/bench_c.err; tail -c 600 gpurun_out/bench_c.json
