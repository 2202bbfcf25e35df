#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "not slow" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for c in c3 c4 c2; do
timeout 900 python scripts/sweep.py --config $c --variants 4,7 --tiers hybrid,global > gpurun_out/sweep_$c.jsonl 2> gpurun_out/sweep_$c.err
done
