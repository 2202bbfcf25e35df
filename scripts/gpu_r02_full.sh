#!/bin/bash
# Round-2 evidence on one B200: build, smoke, the whole GPU suite (incl. full-size parity),
# bench (C3 + C2/C4 extra lines), the reference arm, an ncu launch list of the bench
# command, ncu --set full of the list-mode scan for C3/C2/C4, and the C5 grid.
# scripts/summarize_r02.py copies the results into profiles/.
#   SKIP_EVIDENCE=1  only the C5 grid (SWEEP_LOGN, default 26,28,30,34)
#   SKIP_SWEEP=1     everything but the C5 grid
#   SKIP_TESTS=1     no pytest;  WITH_SANITIZE=1  compute-sanitizer runs too
mkdir -p gpurun_out/full
O=gpurun_out/full
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm,power.limit --format=csv > $O/gpu.txt 2>&1
(nproc; lscpu | head -20) > $O/host.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
if [ "$SKIP_EVIDENCE" != "1" ]; then
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
  if [ "$SKIP_TESTS" != "1" ]; then
    timeout 3000 python -m pytest tests -m gpu -q --durations=40 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
  fi
  timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench.json 2> $O/bench.err
  timeout 900 python bench.py --impl reference --steps 5 --warmup 1 > $O/bench_ref.json 2> $O/bench_ref.err
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv \
    python bench.py --steps 3 --warmup 1 --no-e2e --no-cpu-baseline --extra '' > $O/ncu_bench.out 2>&1
  for c in c3 c2 c4; do
    timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan_staged -s 1 -c 1 \
      -o $O/prof_${c}_list python scripts/prof_target.py --config $c --reps 1 --mode list > $O/ncu_$c.out 2>&1
    # gpurun copies back at most 64 MiB: keep the raw metrics as CSV, the report only for C3
    ncu -i $O/prof_${c}_list.ncu-rep --page raw --csv > $O/prof_${c}_list.raw.csv 2>/dev/null
    [ "$c" != "c3" ] && rm -f $O/prof_${c}_list.ncu-rep
  done
fi
if [ "$SKIP_SWEEP" != "1" ]; then
  # SWEEP_OUT: another file name for a partial re-run (merged by hand); SWEEP_ARGS: extra flags
  timeout 6000 python scripts/sweep_c5.py --logn ${SWEEP_LOGN:-26,28,30,34} --patterns 1000,5000,10000,20000,50000 \
    $SWEEP_ARGS > $O/${SWEEP_OUT:-sweep_c5}.jsonl 2> $O/${SWEEP_OUT:-sweep_c5}.err
fi
if [ "$WITH_SANITIZE" = "1" ]; then
  for tool in memcheck racecheck synccheck initcheck; do
    timeout 600 compute-sanitizer --tool $tool --target-processes all --print-limit 50 --num-cuda-barriers 128 \
      python scripts/sanitize_target.py > $O/sanitize_$tool.log 2>&1
    echo "exit=$?" >> $O/sanitize_$tool.log
  done
fi
