#!/bin/bash
# scratch recipe: SPLIT EVENTS with inline emission (DENSE instantiation)
O=gpurun_out/exp23
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "dense or split or configs_scaled or shard or variants" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 900 python scripts/exp_tiers.py --workloads c5-english-20000-28,c5-english-50000-28 --tiers auto --list --exact-cap >> $O/tiers.jsonl 2>> $O/tiers.err
timeout 600 python scripts/exp_tiers.py --workloads c3 --tiers auto --list >> $O/tiers.jsonl 2>> $O/tiers.err
