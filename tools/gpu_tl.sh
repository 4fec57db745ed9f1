python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python tools/quick_run.py --config c2 --reps 2 2>&1 | grep -v "^gen\|^load" | python -c "
import sys, ast
for line in sys.stdin:
    line=line.strip()
    if line.startswith('{\'t\''):
        d=ast.literal_eval(line); print('t=%2d wall=%7.2f h2d=%7.2f idle=%6.2f static=%6.2f ond=%6.2f cls=%5.2f fin=%5.2f chunks=%3d miss_MB=%8.1f head=%.3f gaps=%.3f tail=%.3f' % (d['t'], d['ms_total'], d['ms_h2d'], d['ms_total']-d['ms_h2d'], d['ms_static'], d['ms_ondemand'], d['ms_classify'], d['ms_finalize'], d['chunks'], d['miss_bytes']/1e6, d['ms_link_head'], d['ms_link_gaps'], d['ms_link_tail']))
    else: print(line[:300])
"
