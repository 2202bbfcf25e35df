#!/bin/bash
# Round-2 check: build, smoke, the GPU suite (FULL=1: incl. full-size parity), bench, tier timings.
mkdir -p gpurun_out/chk
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/chk/build.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/chk/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/chk/smoke.log
timeout 900 python scripts/exp_tiers.py --workloads c3 --tiers split,global --variants 0 > gpurun_out/chk/tiers.jsonl 2> gpurun_out/chk/tiers.err
timeout 900 python scripts/exp_tiers.py --workloads c3 --tiers split,global --variants 0 --list >> gpurun_out/chk/tiers.jsonl 2>> gpurun_out/chk/tiers.err
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/chk/bench.json 2> gpurun_out/chk/bench.err
SEL="gpu and not slow"; [ "$FULL" = "1" ] && SEL="gpu"
timeout 3000 python -m pytest tests -m "$SEL" -q --durations=30 > gpurun_out/chk/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/chk/pytest_gpu.log
