python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
nvidia-smi --query-gpu=pci.bus_id,clocks.sm,pcie.link.gen.current,pcie.link.width.current --format=csv
for r in 1 2; do for v in 0 1; do echo "old=$v"; ASC_GATHER_OLD=$v timeout 600 python tools/quick_run.py --config c2 --reps 3 --quiet 2>&1 | grep -E "kernels" | tail -1 | cut -c1-200; done; done
