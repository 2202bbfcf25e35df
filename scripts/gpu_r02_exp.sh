#!/bin/bash
mkdir -p gpurun_out/exp
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/exp/build.log 2>&1
timeout 300 python scripts/exp_tiers.py --workloads c5-english-5000-28 --tiers auto --variants 0 > gpurun_out/exp/tiers.jsonl 2> gpurun_out/exp/tiers.err
timeout 300 python scripts/exp_tiers.py --workloads c5-english-5000-28 --tiers auto --variants 0 --list --exact-cap >> gpurun_out/exp/tiers.jsonl 2>> gpurun_out/exp/tiers.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_scan_staged -s 2 -c 1 -o gpurun_out/exp/prof_eng_emit python scripts/prof_target.py --config c5-english-5000-28 --reps 1 --mode list > gpurun_out/exp/ncu.out 2>&1
ncu -i gpurun_out/exp/prof_eng_emit.ncu-rep --page raw --csv > gpurun_out/exp/prof_eng_emit.raw.csv 2>/dev/null
ncu -i gpurun_out/exp/prof_eng_emit.ncu-rep --page source --csv --print-source sass > gpurun_out/exp/prof_eng_emit.src.csv 2>/dev/null
rm -f gpurun_out/exp/prof_eng_emit.ncu-rep
