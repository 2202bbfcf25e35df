#!/bin/bash
mkdir -p gpurun_out/exp
AC_EXTRA_NVCC_FLAGS=-DAC_DEBUG_TIMES python -c "
import sys; sys.path.insert(0,'paper_conf_ipps_tranlhc13_b200')
from paper_conf_ipps_tranlhc13_b200 import _build; _build.build(force=True)" > gpurun_out/exp/build.log 2>&1
timeout 600 python scripts/exp_cta_times.py > gpurun_out/exp/cta_times.txt 2>&1
