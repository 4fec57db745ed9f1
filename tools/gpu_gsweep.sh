# gather CTA sweep on C4-shaped (b_e = 4) and C2 (b_e = 8)
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python tools/quick_run.py --config c4 --scale-override 26 --reps 1 --quiet --sweep --sweep-ctas 128,192,256,384,592 --sweep-caps 0 2>&1 | grep gather_ctas
timeout 900 python tools/quick_run.py --config c2 --reps 1 --quiet --sweep --sweep-ctas 64,96,128,192 --sweep-caps 0 2>&1 | grep gather_ctas
