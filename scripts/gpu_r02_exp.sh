#!/bin/bash
mkdir -p gpurun_out/exp
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/exp/build.log 2>&1
for r in 1 2; do
timeout 300 python scripts/exp_tiers.py --workloads c3 --tiers split --variants 0 --list >> gpurun_out/exp/tiers_rewalk.jsonl 2>> gpurun_out/exp/tiers.err
done
AC_EXTRA_NVCC_FLAGS=-DAC_SPLIT_INLINE_EMIT python -c "
from paper_conf_ipps_tranlhc13_b200 import _build; _build.build(force=True)" > gpurun_out/exp/build2.log 2>&1
for r in 1 2; do
timeout 300 python scripts/exp_tiers.py --workloads c3 --tiers split --variants 0 --list >> gpurun_out/exp/tiers_inline.jsonl 2>> gpurun_out/exp/tiers.err
done
