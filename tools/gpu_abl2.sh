python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
ABLATION_ONLY=replace timeout 1500 python tools/ablation.py c2 c4 2>&1 | grep -v "^{" | tail -22
cp gpurun_out/ablation.md gpurun_out/ablation_replace.md
ABLATION_ONLY=prd timeout 1500 python tools/ablation.py c2 c3 2>&1 | grep -v "^{" | tail -12
cp gpurun_out/ablation.md gpurun_out/ablation_prd.md
