#!/bin/bash
# scratch recipe: three-stage event gather pipeline
O=gpurun_out/exp18
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "dense or saturated or configs_scaled or tiers" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 900 python scripts/exp_tiers.py --workloads c5-english-5000-28,c5-english-10000-28,c5-english-20000-28,c5-english-50000-28 --tiers auto --list --exact-cap >> $O/tiers.jsonl 2>> $O/tiers.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_scan_staged|k_gather" -s 1 -c 2 --csv \
     python scripts/prof_target.py --config c5-english-5000-28 --reps 1 --mode list > $O/ncu_ev.csv 2>&1
