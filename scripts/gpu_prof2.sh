#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "not slow" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_staged -s 2 -c 3 -o gpurun_out/prof_c2_compact python scripts/prof_target.py --config c2 --reps 2 > gpurun_out/ncu_full.out 2>&1
