"""Build guard: the hot scan kernels must not spill registers to local
memory (a spill in the 1024-thread staged kernel once cost 1.5x and tripled
its DRAM writes).  Compiles the COMPACT and SMEM tier translation units with
`-Xptxas -v` (nvcc cross-compiles for sm_100a without a GPU)."""
from __future__ import annotations

import re
import shutil
import subprocess
from pathlib import Path

import pytest

from paper_conf_ipps_tranlhc13_b200 import _build

pytestmark = pytest.mark.skipif(shutil.which(_build.nvcc()) is None and not Path(_build.nvcc()).exists(),
                                reason="nvcc not available")


@pytest.mark.parametrize("unit", ["ac_tier_compact.cu"])  # the bench path; one unit keeps the CPU suite short
def test_staged_kernels_do_not_spill(unit, tmp_path):
    cmd = [_build.nvcc(), *_build.CFLAGS, "-Xptxas=-v", f"-I{_build.INCLUDE}", f"-I{_build.CSRC}", "-c",
           str(_build.CSRC / unit), "-o", str(tmp_path / "x.o")]
    out = subprocess.run(cmd, capture_output=True, text=True, check=True).stderr
    bad = []
    cur = None
    for line in out.splitlines():
        m = re.search(r"Compiling entry function '([^']+)'", line)
        if m:
            cur = m.group(1)
        m = re.search(r"(\d+) bytes spill stores", line)
        if m and int(m.group(1)) > 0 and cur and "k_scan_staged" in cur:
            bad.append((cur, int(m.group(1))))
    assert not bad, f"spilling staged kernels: {bad[:5]}"
