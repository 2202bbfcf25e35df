#!/bin/bash
mkdir -p gpurun_out/exp
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/exp/build.log 2>&1
timeout 900 python -m pytest tests -q -m "gpu and not slow" -k "split or c3 or worked or variants" > gpurun_out/exp/pytest.log 2>&1; echo "rc=$?" >> gpurun_out/exp/pytest.log
timeout 900 python scripts/exp_tiers.py --workloads c3 --tiers split --variants 0,10 > gpurun_out/exp/tiers.jsonl 2> gpurun_out/exp/tiers.err
timeout 900 python scripts/exp_tiers.py --workloads c3 --tiers split --variants 0,10 --list >> gpurun_out/exp/tiers.jsonl 2>> gpurun_out/exp/tiers.err
timeout 900 python scripts/exp_tiers.py --workloads c5-snort-1000-28,c5-snort-5000-28,c5-snort-20000-28,c5-snort-50000-28,c5-english-5000-28 --tiers auto,split,global --variants 0 --list >> gpurun_out/exp/tiers.jsonl 2>> gpurun_out/exp/tiers.err
