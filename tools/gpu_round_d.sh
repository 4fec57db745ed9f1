# session D: tests, resident numbers, bench line, bench launch list + ncu captures, resident static-kernel ncu
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -6
timeout 1200 python -m pytest tests -m gpu -q 2>&1 | grep -v "^  File" | tail -4
bash tools/gpu_resident.sh 2>&1 | grep -E "==|kernels" | cut -c1-120
timeout 1200 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err; tail -c 400 gpurun_out/bench_c2.json
mkdir -p gpurun_out/caps && rm -f gpurun_out/caps/*
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/caps/launches.csv \
   python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/bench_ncu.json 2>&1; echo "launch list rc=$?"
for k in k_gather k_ondemand k_static_med k_classify; do
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:$k -s 20 -c 1 -o gpurun_out/caps/prof_$k -f \
     python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1; echo "ncu $k rc=$?"
done
mkdir -p gpurun_out/res && rm -f gpurun_out/res/*
for k in "k_static_med<\(int\)1" "k_static_small<\(int\)1" "k_static_med<\(int\)2" "k_static_hub<\(int\)1"; do
  f=$(echo "$k" | tr -dc 'a-z0-9_')
  timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:$k" -s 4 -c 1 \
     -o gpurun_out/res/prof_$f -f python tools/ncu_new_kernels.py resident > /dev/null 2>&1; echo "ncu resident $k rc=$?"
done
