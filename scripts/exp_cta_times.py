"""Debug experiment: per-warp walk times of the staged SPLIT scan on C3 (needs a
build with AC_EXTRA_NVCC_FLAGS=-DAC_DEBUG_TIMES).  Prints the distribution of
warp walk times and CTA start offsets, count and list mode."""
from __future__ import annotations

import ctypes
import sys
from pathlib import Path

ROOT = Path(__file__).resolve().parents[1]
sys.path.insert(0, str(ROOT))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_tranlhc13_b200 as ac  # noqa: E402
import synth  # noqa: E402


def main():
    w = synth.make("c3")
    stt = ac.build(w.patterns)
    text = torch.from_numpy(w.text).cuda()
    L = ac.lib()
    L.ac_debug_times.argtypes = [ctypes.c_void_p, ctypes.c_uint]
    res = torch.zeros(2, dtype=torch.int64, device="cuda")
    out = torch.empty(w.text.size // 8 + 64, dtype=torch.int64, device="cuda")
    for mode, o in (("count", None), ("list", out), ("count", None), ("list", out)):
        for _ in range(2):
            ac.match_async(stt, text, o, res)
        torch.cuda.synchronize()
        buf = np.zeros(148 * 32 * 2, dtype=np.uint64)
        assert L.ac_debug_times(buf.ctypes.data, buf.size) == 0
        b = buf.reshape(148, 32, 2)
        t0 = b[:, :, 0].astype(np.int64)
        dur = (b[:, :, 1] & ((1 << 48) - 1)).astype(np.int64)
        sm = (b[:, :, 1] >> 48).astype(np.int64)
        start = t0 - t0.min()
        end = start + dur
        cta_end = end.max(axis=1)
        print(mode, "kernel span us", end.max() / 1e3,
              "warp walk us: min/median/max", dur.min() / 1e3, np.median(dur) / 1e3, dur.max() / 1e3,
              "cta start spread us", (t0.min(axis=1).max() - t0.min()) / 1e3,
              "cta end quantiles us", np.percentile(cta_end, [0, 50, 90, 99, 100]) / 1e3, flush=True)
        worst = np.argsort(-cta_end)[:5]
        print("   slowest CTAs (tile, sm, start us, end us):",
              [(int(i), int(sm[i, 0]), start[i].min() / 1e3, cta_end[i] / 1e3) for i in worst], flush=True)


if __name__ == "__main__":
    main()
