# launch list + ncu --set full captures of the bench command (1 GPU)
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
   python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/bench_ncu.json 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_gather -s 40 -c 1 -o gpurun_out/prof_gather -f \
   python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_ondemand -s 40 -c 1 -o gpurun_out/prof_ondemand -f \
   python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_static_med -s 10 -c 1 -o gpurun_out/prof_static_med -f \
   python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_classify -s 20 -c 1 -o gpurun_out/prof_classify -f \
   python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
ls -la gpurun_out/
