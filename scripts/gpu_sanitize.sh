#!/bin/bash
# compute-sanitizer over every scan kernel on small inputs (scripts/sanitize_target.py).
mkdir -p gpurun_out/san
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/san/build.log 2>&1
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1500 compute-sanitizer --tool $tool --target-processes all --print-limit 50 \
    python scripts/sanitize_target.py > gpurun_out/san/$tool.log 2>&1
  echo "exit=$?" >> gpurun_out/san/$tool.log
done
