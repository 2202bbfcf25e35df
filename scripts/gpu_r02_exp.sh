#!/bin/bash
mkdir -p gpurun_out/exp
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/exp/build.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_staged -s 1 -c 1 -o gpurun_out/exp/prof_c3_v7_count python scripts/prof_target.py --config c3 --reps 1 --mode count > gpurun_out/exp/ncu1.out 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_staged -s 1 -c 1 -o gpurun_out/exp/prof_c3_v7_list python scripts/prof_target.py --config c3 --reps 1 --mode list > gpurun_out/exp/ncu2.out 2>&1
