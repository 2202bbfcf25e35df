#!/bin/bash
mkdir -p gpurun_out/p1
(nproc; lscpu | head -20; free -g; nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv) > gpurun_out/p1/host.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/p1/build.log 2>&1
timeout 600 python bench.py --config c3 --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/p1/bench_c3.json 2> gpurun_out/p1/bench_c3.err
timeout 600 python bench.py --config c4 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/p1/bench_c4.json 2> gpurun_out/p1/bench_c4.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_staged -s 1 -c 1 -o gpurun_out/p1/prof_c3_list python scripts/prof_target.py --config c3 --reps 1 --mode list > gpurun_out/p1/ncu_c3.out 2>&1
timeout 300 python -c "
import time, sys; sys.path.insert(0,'.')
import synth
from oracle import Oracle
from concurrent.futures import ThreadPoolExecutor
w = synth.make('c3', n=1<<26)
o = Oracle(w.patterns)
t=time.time(); o.count(w.text[:1<<24]); print('c3 oracle 16MiB 1 thread', time.time()-t, flush=True)
" > gpurun_out/p1/oracle_rate.txt 2>&1
