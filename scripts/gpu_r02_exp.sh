#!/bin/bash
# scratch recipe for the current experiment: emit_coop on/off/batch x staged variants
O=gpurun_out/exp4
mkdir -p $O
LIB=paper_conf_ipps_tranlhc13_b200/libac.so
for v in coop_b1 coop0 coop_b2; do
  cp exp_libs/$v.so $LIB
  timeout 600 python scripts/exp_tiers.py --workloads c5-english-5000-28 --tiers auto --list --exact-cap --variants 0,1,5,9,12 2>> $O/tiers.err | sed "s/^{/{\"lib\": \"$v\", /" >> $O/tiers.jsonl
  timeout 600 python scripts/exp_tiers.py --workloads c5-english-20000-28 --tiers auto --list --exact-cap --variants 0,12 2>> $O/tiers.err | sed "s/^{/{\"lib\": \"$v\", /" >> $O/tiers.jsonl
done
cp exp_libs/coop_b1.so $LIB
timeout 600 python scripts/exp_tiers.py --workloads c3,c2 --tiers auto --list --variants 0,12 2>> $O/tiers.err | sed "s/^{/{\"lib\": \"coop_b1\", /" >> $O/tiers.jsonl
timeout 600 python scripts/exp_tiers.py --workloads c3 --tiers auto --variants 0,12 2>> $O/tiers.err | sed "s/^{/{\"lib\": \"coop_b1\", /" >> $O/tiers.jsonl
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "variants or split" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
