# bench lines C2 (default), C3, C4 + launch list and ncu captures of the C2 bench command
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err; cut -c1-200 gpurun_out/bench_c2.json
timeout 1500 python bench.py --config c3 --steps 3 > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err; cut -c1-200 gpurun_out/bench_c3.json
timeout 1500 python bench.py --config c4 --steps 3 > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err; cut -c1-200 gpurun_out/bench_c4.json
bash tools/gpu_profile.sh > /dev/null 2>&1
ls gpurun_out | head -30
