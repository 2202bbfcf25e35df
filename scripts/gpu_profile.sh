#!/bin/bash
# bench + ncu launch list + one full ncu capture of the staged scan (C2)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "not slow" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 50 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 3 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_bench.out 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_staged -s 2 -c 2 -o gpurun_out/prof_c2 python scripts/prof_target.py --config c2 --reps 2 > gpurun_out/ncu_full.out 2>&1
