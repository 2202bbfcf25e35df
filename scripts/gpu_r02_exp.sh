#!/bin/bash
# scratch recipe: check the planner change on the big/adversarial points + bench
O=gpurun_out/exp14
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_abi.py -q -x -k "not slow" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err
timeout 2400 python scripts/sweep_c5.py --logn 34 --families adv --big english-1000 > $O/sweep.jsonl 2> $O/sweep.err
