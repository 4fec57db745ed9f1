timeout 900 python tools/quick_run.py --config c2 --reps 1 --sweep --quiet 2>&1 | tail -20
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gather -s 30 -c 2 -o gpurun_out/prof_gather2 -f python tools/quick_run.py --config c2 --reps 1 --quiet > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_ondemand -s 30 -c 2 -o gpurun_out/prof_ondemand2 -f python tools/quick_run.py --config c2 --reps 1 --quiet > /dev/null 2>&1
