#!/bin/bash
# scratch recipe: EVENTS on 16-bit tables (adversarial C5 points)
O=gpurun_out/exp15
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_abi.py -q -x -k "not slow" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 1200 python scripts/sweep_c5.py --logn 26 --families adv --patterns 1000 --big none > $O/sweep.jsonl 2> $O/sweep.err
timeout 600 python scripts/exp_tiers.py --workloads c5-english-5000-28,c5-english-20000-28 --tiers auto --list --exact-cap >> $O/tiers.jsonl 2>> $O/tiers.err
timeout 600 python scripts/exp_tiers.py --workloads c2,c3,c1 --tiers auto --list >> $O/tiers.jsonl 2>> $O/tiers.err
