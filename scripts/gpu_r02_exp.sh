#!/bin/bash
mkdir -p gpurun_out/exp
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/exp/build.log 2>&1
timeout 300 python -m pytest tests -q -x -m "gpu and not slow" -k "split or c3 or worked or variants or snort" > gpurun_out/exp/pytest.log 2>&1; echo "rc=$?" >> gpurun_out/exp/pytest.log
timeout 200 python scripts/exp_tiers.py --workloads c3 --tiers split --variants 10,7 > gpurun_out/exp/tiers.jsonl 2> gpurun_out/exp/tiers.err
timeout 200 python scripts/exp_tiers.py --workloads c3 --tiers split --variants 10,7 --list >> gpurun_out/exp/tiers.jsonl 2>> gpurun_out/exp/tiers.err
timeout 200 python scripts/exp_tiers.py --workloads c2 --tiers auto --variants 0 --list >> gpurun_out/exp/tiers.jsonl 2>> gpurun_out/exp/tiers.err
timeout 200 python scripts/exp_tiers.py --workloads c2 --tiers auto --variants 0 --list --exact-cap >> gpurun_out/exp/tiers.jsonl 2>> gpurun_out/exp/tiers.err
