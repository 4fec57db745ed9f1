python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python tools/quick_run.py --config c2 --reps 1 --quiet --sweep --sweep-ctas 64,128,192,256,384 --sweep-caps 0 2>&1 | grep gather_ctas
timeout 900 python tools/quick_run.py --config c4 --scale-override 26 --reps 1 --quiet --sweep --sweep-ctas 128,256,384,512 --sweep-caps 0 2>&1 | grep gather_ctas
