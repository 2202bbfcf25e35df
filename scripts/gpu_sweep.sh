#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "not slow" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python scripts/sweep.py --config c4 --variants 4,7 > gpurun_out/sweep_c4.jsonl 2> gpurun_out/sweep_c4.err
timeout 900 python -m pytest tests -m gpu -x -q -k "full_size_sampled and c4" > gpurun_out/pytest_c4full.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_c4full.log
