#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "not slow" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python scripts/sweep.py --config c1 --n 268435456 --variants 1,2,3,4,5,6 --global-kernel > gpurun_out/sweep_c1big.jsonl 2> gpurun_out/sweep_c1big.err
for c in c2 c3 c4; do
  timeout 600 python scripts/sweep.py --config $c --variants 1,2,3,4,5,6 --global-kernel --tiers auto,global > gpurun_out/sweep_$c.jsonl 2> gpurun_out/sweep_$c.err
done
