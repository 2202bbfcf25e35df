#!/bin/bash
# scratch recipe: evict-first event stores, staged vs direct
O=gpurun_out/exp13
mkdir -p $O
LIB=paper_conf_ipps_tranlhc13_b200/libac.so
for v in stage nostage; do
  cp exp_libs/$v.so $LIB
  timeout 900 python scripts/exp_tiers.py --workloads c5-english-5000-28,c5-english-10000-28,c5-english-20000-28,c5-english-50000-28 --tiers auto --list --exact-cap 2>> $O/tiers.err | sed "s/^{/{\"lib\": \"$v\", /" >> $O/tiers.jsonl
  timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"k_scan_staged|k_gather" -s 1 -c 2 --csv \
     python scripts/prof_target.py --config c5-english-5000-28 --reps 1 --mode list > $O/ncu_$v.csv 2>&1
done
cp exp_libs/stage.so $LIB
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "dense or configs_scaled or split or stride2 or tiers" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
