# one gpurun call: tests, bench, reference arm, ncu launch list, ncu full captures
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -c 3000 gpurun_out/bench.json
timeout 900 python bench.py --impl reference > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; cat gpurun_out/bench_ref.json
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
   python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/bench_ncu.json 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_gather -s 20 -c 2 -o gpurun_out/prof_gather -f \
   python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_ondemand -s 20 -c 2 -o gpurun_out/prof_ondemand -f \
   python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_static -s 20 -c 3 -o gpurun_out/prof_static -f \
   python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 0 > /dev/null 2>&1
ls -la gpurun_out
