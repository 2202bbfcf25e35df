#!/bin/bash
# scratch recipe: EVENTS gather pipelining
O=gpurun_out/exp9
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "dense or tiers or configs_scaled or worked or c1 or split or stride2 or misaligned or edge" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 900 python scripts/exp_tiers.py --workloads c5-english-5000-28,c5-english-10000-28,c5-english-20000-28,c5-english-50000-28 --tiers auto --list --exact-cap --two-pass 0,1 >> $O/tiers.jsonl 2>> $O/tiers.err
timeout 600 python scripts/exp_tiers.py --workloads c2,c3 --tiers auto --list >> $O/tiers.jsonl 2>> $O/tiers.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_e5k.csv \
  python scripts/prof_target.py --config c5-english-5000-28 --reps 2 --mode list > $O/ncu_l.out 2>&1
timeout 900 ncu --set full --clock-control none -k regex:k_gather -c 1 \
  -o $O/prof_gather python scripts/prof_target.py --config c5-english-5000-28 --reps 1 --mode list > $O/ncu_g.out 2>&1
ncu -i $O/prof_gather.ncu-rep --page raw --csv > $O/prof_gather.raw.csv 2>/dev/null
rm -f $O/prof_gather.ncu-rep
