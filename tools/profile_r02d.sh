#!/bin/bash
# Round-2d evidence (GPU box, repo root; gpurun_out/prof3/): ncu --set full of the CSR build kernels
# after the radix-pass instruction cuts (three-instruction digit peers, DEG-specialised last pass)
set -x
O=gpurun_out/prof3
mkdir -p $O
timeout 900 ncu --clock-control none --set full --import-source on -k 'regex:k_onesweep|k_coo_scan|k_place' -o $O/build \
    python tools/build_probe.py --reps 0 > $O/build.log 2>&1
python tools/ncu_summary.py $O/build.ncu-rep > $O/build_summary.txt 2>&1
rm -f $O/build.ncu-rep
timeout 300 python tools/build_probe.py --reps 9 > $O/build_times.txt 2>&1
timeout 300 python tools/build_probe.py --reps 5 --sym 1 >> $O/build_times.txt 2>&1
timeout 300 python tools/build_probe.py --reps 5 --weighted 1 >> $O/build_times.txt 2>&1
timeout 300 python tools/build_probe.py --reps 5 --host 1 >> $O/build_times.txt 2>&1
