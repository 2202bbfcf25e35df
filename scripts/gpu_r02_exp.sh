#!/bin/bash
# scratch recipe: check the final emission configuration
O=gpurun_out/exp6
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 600 python scripts/exp_tiers.py --workloads c5-english-1000-28,c5-english-5000-28,c5-english-10000-28,c5-english-20000-28 --tiers auto --list --exact-cap >> $O/tiers.jsonl 2>> $O/tiers.err
timeout 600 python scripts/exp_tiers.py --workloads c3,c2 --tiers auto --list >> $O/tiers.jsonl 2>> $O/tiers.err
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "dense or variants or split or tiers or compact" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
