#!/bin/bash
# scratch recipe: per-state output counts in shared memory for the staged GLOBAL scan
O=gpurun_out/exp22
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "dense or tiers or configs_scaled or saturated or stride2 or worked or c1 or shard" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 900 python scripts/exp_tiers.py --workloads c5-english-5000-28,c5-english-10000-28 --tiers auto --list --exact-cap >> $O/tiers.jsonl 2>> $O/tiers.err
timeout 900 python scripts/exp_tiers.py --workloads c5-english-5000-28,c5-english-10000-28,c5-snort-1000-28,c5-snort-50000-28 --tiers auto >> $O/tiers.jsonl 2>> $O/tiers.err
timeout 600 python scripts/exp_tiers.py --workloads c4 --n 4294967296 --tiers auto --list >> $O/tiers.jsonl 2>> $O/tiers.err
