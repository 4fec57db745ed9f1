# end-of-round evidence: build + smoke + GPU suite, bench lines C2 (default) / C3 / C4, launch list and ncu captures
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 1500 python -m pytest tests -m gpu -q 2>&1 | tail -2
timeout 900 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err; cut -c1-160 gpurun_out/bench_c2.json
timeout 1500 python bench.py --config c3 --steps 3 > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err; cut -c1-160 gpurun_out/bench_c3.json
timeout 1500 python bench.py --config c4 --steps 3 > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err; cut -c1-160 gpurun_out/bench_c4.json
timeout 600 python bench.py --impl reference > gpurun_out/bench_ref_c2.json 2>/dev/null; cut -c1-160 gpurun_out/bench_ref_c2.json
bash tools/gpu_profile.sh > /dev/null 2>&1
ls gpurun_out | wc -l
