#!/bin/bash
# Full ncu capture of the staged scan on C2: the count launch and the first list-mode launch.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_staged -s 0 -c 2 -o gpurun_out/prof_c2_${1:-cur} python scripts/prof_target.py --config c2 --reps 1 > gpurun_out/ncu_full.out 2>&1
echo "ncu rc=$?" >> gpurun_out/ncu_full.out
