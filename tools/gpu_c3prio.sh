# C3 (PR, 6 iterations): compute-stream priority and static CTAs/SM vs the per-iteration slow on-demand kernel
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
for v in "ASC_CS_PRI_UP=0" "ASC_CS_PRI_UP=1" "ASC_CS_PRI_UP=2"; do
  echo "== c3 [$v]"
  env $v ASCETIC_TRACE=1 timeout 900 python tools/quick_run.py --config c3 --iters 6 --reps 2 --quiet --static-ctas 4,2,6 2> gpurun_out/c3p_${v}.txt | grep -E "static_ctas|kernels" | cut -c1-250
done
python -c "import torch; print(torch.cuda.get_device_properties(0)); import ctypes" ; nvidia-smi -q | grep -i -A3 "priority" | head
