#!/bin/bash
# Round-2 evidence pass (run on a GPU box from the repo root; writes gpurun_out/prof/):
#   1. ncu launch list of the bench command (per-launch device time, serialised, cold cache)
#   2. ncu --set full of every frontier relax launch (canonical ids), summarised on the box
#   3. ncu --set full of one PageRank relax launch (the dominant kernel) -> .ncu-rep + summary
#   4. ncu --set full of the CSR build kernels (second of two device-input builds)
#   5. ncu launch list of a host-input build (the sorted-runs path)
set -x
O=gpurun_out/prof
mkdir -p $O
NCU="ncu --clock-control none"
timeout 900 $NCU --metrics gpu__time_duration.sum --csv --log-file $O/launches_bench.csv \
    python bench.py --steps 2 --warmup 3 --no-configs > $O/launches_bench.log 2>&1
python tools/launches.py $O/launches_bench.csv > $O/launches_bench_summary.txt
timeout 900 $NCU --set full -k regex:k_relax_fq -o $O/frontier \
    python tools/frontier_probe.py --reps 0 --graph 0 > $O/frontier.log 2>&1
python tools/ncu_summary.py $O/frontier.ncu-rep > $O/frontier_summary.txt 2>&1
rm -f $O/frontier.ncu-rep
timeout 600 $NCU --set full --import-source on -k regex:k_relax_pr_cid -s 5 -c 1 -o $O/relax_pr \
    python bench.py --profile --steps 1 --warmup 0 --no-cpu > $O/relax_pr.log 2>&1
python tools/ncu_summary.py $O/relax_pr.ncu-rep > $O/relax_pr_summary.txt 2>&1
timeout 900 $NCU --set full -k 'regex:k_onesweep|k_coo_scan|k_place|k_digit' -o $O/build \
    python tools/build_probe.py --reps 0 > $O/build.log 2>&1
python tools/ncu_summary.py $O/build.ncu-rep > $O/build_summary.txt 2>&1
rm -f $O/build.ncu-rep
timeout 600 $NCU --metrics gpu__time_duration.sum --csv --log-file $O/launches_hostbuild.csv \
    python tools/build_probe.py --host 1 --reps 0 > $O/hostbuild.log 2>&1
python tools/launches.py $O/launches_hostbuild.csv > $O/launches_hostbuild_summary.txt
