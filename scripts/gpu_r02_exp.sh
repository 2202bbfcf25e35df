#!/bin/bash
# scratch recipe: split_next trims + identity class map instantiation
O=gpurun_out/exp7
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for r in 1 2; do
timeout 600 python scripts/exp_tiers.py --workloads c3 --tiers auto --list >> $O/tiers.jsonl 2>> $O/tiers.err
timeout 600 python scripts/exp_tiers.py --workloads c3 --tiers auto >> $O/tiers.jsonl 2>> $O/tiers.err
done
timeout 600 python scripts/exp_tiers.py --workloads c5-english-20000-28 --tiers auto --list --exact-cap >> $O/tiers.jsonl 2>> $O/tiers.err
timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "split or configs_scaled or dense or variants" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
