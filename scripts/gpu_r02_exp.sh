#!/bin/bash
# evidence: ncu --set full of the EVENTS single pass (scan + gather) on C5 English 5K, 256 MiB
O=gpurun_out/events
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:"k_scan_staged|k_gather" -s 1 -c 2 \
  -o $O/prof_ev python scripts/prof_target.py --config c5-english-5000-28 --reps 1 --mode list > $O/ncu_ev.out 2>&1
ncu -i $O/prof_ev.ncu-rep --page raw --csv > $O/prof_ev.raw.csv 2>/dev/null
rm -f $O/prof_ev.ncu-rep
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_ev.csv \
  python scripts/prof_target.py --config c5-english-5000-28 --reps 2 --mode list > $O/ncu_l.out 2>&1
