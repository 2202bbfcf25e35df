#!/bin/bash
# scratch recipe: compile-time row stride in the identity-map SPLIT walk
O=gpurun_out/exp17
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "split or configs_scaled or worked or c3" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
for r in 1 2; do timeout 600 python scripts/exp_tiers.py --workloads c3 --tiers auto --list >> $O/tiers.jsonl 2>> $O/tiers.err; done
timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err
