# §3.4 replacement study on C2 and C4 (tools/ablation.py, ABLATION_ONLY=replace)
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
ABLATION_ONLY=replace timeout 2400 python tools/ablation.py c2 c4 2>&1 | tail -40
cp gpurun_out/ablation.md gpurun_out/ablation_replace.md
