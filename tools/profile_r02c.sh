#!/bin/bash
# Round-2c evidence pass (GPU box, repo root; writes gpurun_out/prof2/): full GPU tests, the bench
# line, the bench's launch list, and full ncu captures of the kernels changed since round 2b
# (k_compact, k_init: frontier loop; k_place_runs: host-input build).
set -x
O=gpurun_out/prof2
mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q > $O/gputests.log 2>&1
( time timeout 900 python bench.py > $O/bench.json 2> $O/bench.err ) 2> $O/bench_time.txt
NCU="ncu --clock-control none"
timeout 900 $NCU --metrics gpu__time_duration.sum --csv --log-file $O/launches_bench.csv \
    python bench.py --steps 2 --warmup 3 --no-configs > $O/launches_bench.log 2>&1
python tools/launches.py $O/launches_bench.csv > $O/launches_bench_summary.txt
timeout 600 $NCU --set full -k 'regex:k_compact|k_init' -o $O/loop \
    python tools/frontier_probe.py --algos bfs --reps 0 --graph 0 > $O/loop.log 2>&1
python tools/ncu_summary.py $O/loop.ncu-rep > $O/loop_summary.txt 2>&1
rm -f $O/loop.ncu-rep
timeout 600 $NCU --set full -k 'regex:k_place_runs|k_pad_runs|k_run_delta' -c 4 -o $O/runs \
    python tools/build_probe.py --host 1 --reps 0 > $O/runs.log 2>&1
python tools/ncu_summary.py $O/runs.ncu-rep > $O/runs_summary.txt 2>&1
rm -f $O/runs.ncu-rep
