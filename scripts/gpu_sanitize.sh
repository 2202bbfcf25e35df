#!/bin/bash
# compute-sanitizer over every scan kernel on small inputs (scripts/sanitize_target.py).
mkdir -p gpurun_out/san
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/san/build.log 2>&1
for tool in memcheck racecheck synccheck initcheck; do
  timeout 600 compute-sanitizer --tool $tool --target-processes all --print-limit 50 --num-cuda-barriers 128 \
    python scripts/sanitize_target.py > gpurun_out/san/$tool.log 2>&1
  echo "exit=$?" >> gpurun_out/san/$tool.log
done
# experiment riding along: variant 11 (32-byte unswizzled single slot) on C2/C3
timeout 300 python scripts/exp_tiers.py --workloads c2 --tiers auto --variants 0,11 --list > gpurun_out/san/tiers.jsonl 2> gpurun_out/san/tiers.err
timeout 300 python scripts/exp_tiers.py --workloads c3 --tiers split --variants 10,11 --list >> gpurun_out/san/tiers.jsonl 2>> gpurun_out/san/tiers.err
timeout 300 python -m pytest tests -q -x -m "gpu and not slow" -k "variants or compact" > gpurun_out/san/pytest.log 2>&1; echo "rc=$?" >> gpurun_out/san/pytest.log
