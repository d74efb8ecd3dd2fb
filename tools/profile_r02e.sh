#!/bin/bash
# Round-2e evidence (GPU box, repo root; gpurun_out/prof4/): the PageRank relax after the
# 1024-thread shape (full ncu capture -> relax_pr_traffic.json), the bench's launch list
set -x
O=gpurun_out/prof4
mkdir -p $O
timeout 600 ncu --clock-control none --set full --import-source on -k regex:k_relax_pr_cid -s 5 -c 1 -o $O/relax_pr \
    python bench.py --profile --steps 1 --warmup 0 --no-cpu > $O/relax_pr.log 2>&1
python tools/ncu_summary.py $O/relax_pr.ncu-rep > $O/relax_pr_summary.txt 2>&1
timeout 900 ncu --clock-control none --metrics gpu__time_duration.sum --csv --log-file $O/launches_bench.csv \
    python bench.py --steps 2 --warmup 3 --no-configs > $O/launches_bench.log 2>&1
python tools/launches.py $O/launches_bench.csv > $O/launches_bench_summary.txt
