#!/bin/bash
mkdir -p gpurun_out/exp
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/exp/build.log 2>&1
timeout 400 python -m pytest tests -q -x -m "gpu and not slow" > gpurun_out/exp/pytest.log 2>&1; echo "rc=$?" >> gpurun_out/exp/pytest.log
timeout 300 python scripts/exp_tiers.py --workloads c5-english-5000-28,c5-english-20000-28 --tiers auto,global --variants 0 --list --exact-cap > gpurun_out/exp/tiers.jsonl 2> gpurun_out/exp/tiers.err
timeout 300 python scripts/exp_tiers.py --workloads c3,c1 --tiers auto --variants 0 --list >> gpurun_out/exp/tiers.jsonl 2>> gpurun_out/exp/tiers.err
