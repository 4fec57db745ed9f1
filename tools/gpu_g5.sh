# same box: old gather / 16-byte gather / 16-byte gather with L1::no_allocate, C2 and C4-shaped
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
nvidia-smi --query-gpu=pci.bus_id --format=csv,noheader
cp paper_conf_icpp_tangzwgzwy21_b200/libascetic.so /tmp/lib_default.so
ASCETIC_NVCC_EXTRA=-DASC_GATHER_NO_ALLOC python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
cp paper_conf_icpp_tangzwgzwy21_b200/libascetic.so /tmp/lib_na.so
for cfg in "c2" "c4 --scale-override 26"; do
  for v in old new na; do
    if [ $v = na ]; then cp /tmp/lib_na.so paper_conf_icpp_tangzwgzwy21_b200/libascetic.so; else cp /tmp/lib_default.so paper_conf_icpp_tangzwgzwy21_b200/libascetic.so; fi
    o=0; [ $v = old ] && o=1
    echo "$cfg $v"; ASC_GATHER_OLD=$o timeout 600 python tools/quick_run.py --config $cfg --reps 3 --quiet 2>&1 | grep -E "kernels" | tail -1 | cut -c1-200
  done
done
cp /tmp/lib_default.so paper_conf_icpp_tangzwgzwy21_b200/libascetic.so
