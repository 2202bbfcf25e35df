#!/bin/bash
# scratch recipe: DSMEM lookup microbenchmark + ncu of the EVENTS single pass
O=gpurun_out/exp10
mkdir -p $O
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o $O/dsmem_bench scripts/dsmem_bench.cu > $O/dsmem_build.log 2>&1
timeout 120 $O/dsmem_bench > $O/dsmem_bench.jsonl 2> $O/dsmem_bench.err
rm -f $O/dsmem_bench
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_scan_staged|k_gather" -s 1 -c 2 \
  -o $O/prof_ev python scripts/prof_target.py --config c5-english-5000-28 --reps 1 --mode list > $O/ncu_ev.out 2>&1
ncu -i $O/prof_ev.ncu-rep --page raw --csv > $O/prof_ev.raw.csv 2>/dev/null
ncu -i $O/prof_ev.ncu-rep --page source --csv --print-source sass > $O/prof_ev.src.csv 2>/dev/null
rm -f $O/prof_ev.ncu-rep
