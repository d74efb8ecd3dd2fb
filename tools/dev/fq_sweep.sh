# frontier relax: FRONTIER_AUTO switch point (TIGR_FQ_DIV) x graph order, cfg4
for r in 0 1; do for d in 1 2 4 16 1000000; do echo "div=$d reorder=$r"; TIGR_FQ_DIV=$d python tools/frontier_probe.py --reps 5 --reorder $r | grep -v reorder_ms; done; done
