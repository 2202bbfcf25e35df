#!/bin/bash
# Round evidence: all GPU tests (incl. full-size), bench, sweeps, ncu launch list and one full capture.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm,power.limit --format=csv > gpurun_out/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_full.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu_full.log
timeout 600 python bench.py --steps 50 --warmup 5 > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 900 python bench.py --impl reference --steps 5 --warmup 1 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
for c in c1 c3 c4; do
  timeout 900 python scripts/sweep.py --config $c --variants 4,7 --global-kernel > gpurun_out/sweep_$c.jsonl 2> gpurun_out/sweep_$c.err
done
timeout 600 python scripts/sweep.py --config c2 --variants 7 --global-kernel --tiers compact,global > gpurun_out/sweep_c2.jsonl 2> gpurun_out/sweep_c2.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 3 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_bench.out 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_staged -s 2 -c 2 -o gpurun_out/prof_c2_full python scripts/prof_target.py --config c2 --reps 2 > gpurun_out/ncu_full.out 2>&1
bash scripts/gpu_ncu_list.sh
