#!/bin/bash
mkdir -p gpurun_out/exp
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/exp/build.log 2>&1
timeout 900 python -m pytest tests -q -m "gpu and not slow" -k "split or c3 or worked" > gpurun_out/exp/pytest.log 2>&1; echo "rc=$?" >> gpurun_out/exp/pytest.log
timeout 900 python scripts/exp_tiers.py --workloads c3 --tiers split --variants 0 --policies 0:0,0:2 > gpurun_out/exp/tiers.jsonl 2> gpurun_out/exp/tiers.err
timeout 900 python scripts/exp_tiers.py --workloads c3,c5-snort-50000-28,c5-english-5000-28 --tiers split,global --variants 0 --policies 0:0,0:2 --list >> gpurun_out/exp/tiers.jsonl 2>> gpurun_out/exp/tiers.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_staged -s 1 -c 1 -o gpurun_out/exp/prof_c3_split5_list python scripts/prof_target.py --config c3 --reps 1 --mode list > gpurun_out/exp/ncu2.out 2>&1
