#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "not slow" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python scripts/sweep.py --config c2 --variants 7 --tiers compact,global > gpurun_out/sweep_c2.jsonl 2> gpurun_out/sweep_c2.err
timeout 600 python scripts/sweep.py --config c1 --n 268435456 --variants 4 > gpurun_out/sweep_c1big.jsonl 2> gpurun_out/sweep_c1big.err
timeout 600 python scripts/sweep.py --config c3 --variants 4 > gpurun_out/sweep_c3.jsonl 2> gpurun_out/sweep_c3.err
