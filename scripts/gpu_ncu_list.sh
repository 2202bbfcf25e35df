#!/bin/bash
# ncu --set full of the C2 list-mode step's kernels (scan + gather).
mkdir -p gpurun_out
[ -f paper_conf_ipps_tranlhc13_b200/libac.so ] || python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_scan_staged|k_gather" -c 5 \
  -o gpurun_out/prof_c2_list python scripts/prof_target.py --config c2 --reps 2 > gpurun_out/ncu_list.out 2>&1
echo "ncu rc=$?" >> gpurun_out/ncu_list.out
