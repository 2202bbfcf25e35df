#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python scripts/sweep.py --config c2 --variants 7,9 --tiers compact > gpurun_out/sweep_c2.jsonl 2> gpurun_out/sweep_c2.err
timeout 900 ncu --set full --clock-control none -k regex:k_scan_staged -s 1 -c 1 -o gpurun_out/prof_c3_count python scripts/prof_target.py --config c3 --reps 1 --mode count > gpurun_out/ncu_c3.out 2>&1
timeout 900 ncu --set full --clock-control none -k regex:k_scan_staged -s 1 -c 1 -o gpurun_out/prof_c4_count python scripts/prof_target.py --config c4 --reps 1 --mode count > gpurun_out/ncu_c4.out 2>&1
