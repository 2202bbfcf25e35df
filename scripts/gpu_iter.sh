#!/bin/bash
# Iteration run: quick parity tests, bench, and a C2 list-mode placement comparison.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "not slow" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err
timeout 600 python scripts/sweep.py --config c2 --variants 7 --two-pass 0,3 > gpurun_out/sweep_gather.jsonl 2> gpurun_out/sweep_gather.err
