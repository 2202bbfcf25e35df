#!/bin/bash
# C3/C4 sweeps only (GLOBAL tier experiments)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "not slow" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for c in c3 c4; do
  timeout 900 python scripts/sweep.py --config $c --variants 4 --global-kernel "$@" > gpurun_out/sweep_$c.jsonl 2> gpurun_out/sweep_$c.err
done
timeout 600 python scripts/sweep.py --config c2 --variants 7 > gpurun_out/sweep_c2.jsonl 2> gpurun_out/sweep_c2.err
