#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python scripts/sweep.py --config c2 --variants 7,4 --tiers compact > gpurun_out/sweep_c2.jsonl 2> gpurun_out/sweep_c2.err
timeout 600 python scripts/sweep.py --config c1 --variants 4 > gpurun_out/sweep_c1.jsonl 2> gpurun_out/sweep_c1.err
timeout 600 python bench.py --steps 30 --warmup 5 --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err
