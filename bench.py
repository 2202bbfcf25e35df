#!/usr/bin/env python
"""bench.py -- input-text Gbps of the Aho-Corasick matching scan on B200.

One step = one pass of the whole hot path over one
shard of synthetic text: ac_match_async in list mode (single emitting scan
into per-chain scratch slots with the chain offsets computed in its epilogue
-> gather into the canonical list in HBM -> overflow re-walk), plus the
count all-reduce across ranks when N > 1.  The STT build and the host->device
copy of the text are outside the timed region, as in the paper.

Workload at N=1: BASELINE.json configs[1] (C2) -- 1,000 patterns of length
4-32 taken from 256 MiB of English-like text.  At N>1 each rank scans its own
256 MiB segment of the same text stream plus a (maxlen-1)-byte halo of the
next segment (weak scaling, per-rank work fixed).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

Prints ONE JSON line (rank 0).  The `--impl reference` arm times the CPU
oracle (oracle/, the only other place this file executes it) on bounded
samples of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import threading
import time
from pathlib import Path

import numpy as np

ROOT = Path(__file__).resolve().parent
sys.path.insert(0, str(ROOT))

METRIC = "input-text Gbps at 1/2/4/8 B200 (device-timed) + fraction of HBM/L1 roofline"
WORKLOADS = {
    "c1": "100 random patterns (len 2-16, alphabet 26) over 1 MiB seeded random lowercase text",
    "c2": "1,000 patterns (len 4-32) over 256 MiB English-like text",
    "c3": "Snort-like 10,000 byte patterns (alphabet 256) over 1 GiB packet-payload text",
    "c4": "DNA: 20,000 k-mers (len 20-32, alphabet 4) over 4 GiB genome-like text",
}
FALLBACK_HBM_GBS = 6650.0


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=50)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", choices=["ours", "reference"], default="ours")
    p.add_argument("--config", default="c2", choices=sorted(WORKLOADS))
    p.add_argument("--mode", default="list", choices=["list", "count"])
    p.add_argument("--kernel", default="auto", choices=["auto", "staged", "global"])
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-e2e", action="store_true")
    return p.parse_args()


def peaks():
    f = ROOT / "MEASURED_PEAKS.json"
    if f.exists():
        d = json.loads(f.read_text())
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)", d
    return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)", {}


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """Samples SM clock and throttle reasons through NVML while running."""

    REASONS = {0x8: "hw_slowdown", 0x40: "hw_thermal_slowdown", 0x20: "sw_thermal_slowdown",
               0x4: "sw_power_cap", 0x80: "hw_power_brake_slowdown", 0x1: "gpu_idle"}

    def __init__(self, index: int):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self._nv = pynvml
            self._h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self._h, pynvml.NVML_CLOCK_SM)
        except Exception as e:  # pragma: no cover
            log("nvml unavailable:", e)
            self._nv = None
        self._t = threading.Thread(target=self._run, daemon=True)

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self._nv.nvmlDeviceGetClockInfo(self._h, self._nv.NVML_CLOCK_SM))
                r = self._nv.nvmlDeviceGetCurrentClocksEventReasons(self._h)
                for bit, name in self.REASONS.items():
                    if r & bit and bit != 0x1:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.005)

    def __enter__(self):
        if self._nv:
            self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._nv:
            self._t.join()

    def summary(self):
        return {"sm_mhz": float(np.median(self.samples)) if self.samples else None, "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


# --------------------------------------------------------------- workload
def load_workload(cfg: str, rank: int, world: int = 1):
    """Rank r scans bytes [r*n, (r+1)*n) of the config's text stream, plus
    the (maxlen-1)-byte halo of the next segment when world > 1."""
    import synth
    t0 = time.time()
    w = synth.make(cfg)
    maxlen = max(len(p) for p in w.patterns)
    halo = maxlen - 1 if world > 1 else 0
    if rank == 0:
        text = w.text
        if halo:
            text = np.concatenate([w.text, synth.stream(w, cfg, w.text.size // synth.BLOCK, halo)])
    else:
        text = synth.segment(w, cfg, rank, w.text.size, halo)
    log(f"[rank {rank}] workload {cfg}: {w.text.size} B, {len(w.patterns)} patterns, gen {time.time() - t0:.1f}s")
    return w, text, halo


# ------------------------------------------------------------ reference arm
def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    from oracle import Oracle
    w, text, _ = load_workload(args.config, 0)
    n = w.text.size
    o = Oracle(w.patterns)
    probe = min(n, 1 << 20)
    t0 = time.perf_counter()
    o.match(text[:probe])
    rate = probe / max(1e-6, time.perf_counter() - t0)
    per_step = int(min(n, max(1 << 16, rate * 90.0 / max(1, args.steps + args.warmup))))
    rng = np.random.default_rng(0)
    los = rng.integers(0, max(1, n - per_step), size=args.steps + args.warmup)
    tot_b, tot_t, cnt = 0, 0.0, 0
    for i, lo in enumerate(los):
        t0 = time.perf_counter()
        ends, _ = o.match(text[lo:lo + per_step])
        dt = time.perf_counter() - t0
        if i >= args.warmup:
            tot_b += per_step
            tot_t += dt
            cnt += ends.size
    gbps = tot_b * 8 / tot_t / 1e9
    sample = f"{args.steps} windows of {per_step} B at seeded offsets of the {args.config} text, 1 thread, build excluded"
    line = {
        "impl": "reference", "metric": METRIC, "value": gbps, "unit": "Gbps", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": tot_t / args.steps * 1e3,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u8", "data": "synthetic",
        "config": {"workload": WORKLOADS[args.config], "mode": "list", "sample_bytes_per_step": per_step},
        "cpu_baseline": {"value": gbps, "unit": "Gbps", "cores": 1, "kind": "oracle", "sample": sample},
        "e2e": {"value": gbps, "unit": "Gbps", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "matches_in_sample": int(cnt),
    }
    print(json.dumps(line), flush=True)
    return 0


def cpu_baseline(w, seconds=12.0):
    from oracle import Oracle
    o = Oracle(w.patterns)
    probe = min(w.text.size, 1 << 20)
    t0 = time.perf_counter()
    o.match(w.text[:probe])
    rate = probe / max(1e-6, time.perf_counter() - t0)
    size = int(min(w.text.size, max(probe, rate * seconds)))
    t0 = time.perf_counter()
    o.match(w.text[:size])
    dt = time.perf_counter() - t0
    return {"value": size * 8 / dt / 1e9, "unit": "Gbps", "cores": 1, "kind": "oracle",
            "sample": f"first {size} B of the text (canonical list), 1 thread, build excluded, {dt:.1f} s"}


# ---------------------------------------------------------------- our arm
def run_ours(args):
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_tranlhc13_b200 as ac

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)
    w, text_np, halo = load_workload(args.config, rank, world)
    n = w.text.size
    stt = ac.build(w.patterns, device=local)
    text = torch.from_numpy(text_np).to(dev)
    base = rank * n
    kernel = {"auto": ac.KERNEL_AUTO, "staged": ac.KERNEL_STAGED, "global": ac.KERNEL_GLOBAL}[args.kernel]
    res = torch.zeros(2, dtype=torch.int64, device=dev)
    ac.match_async(stt, text, None, res, n_halo=halo, base=base, kernel=kernel)
    count = int(res[0].item())
    out = torch.empty(max(1, count), dtype=torch.int64, device=dev) if args.mode == "list" else None
    stream = torch.cuda.current_stream()

    def step():
        k = ac.match_async(stt, text, out, res, n_halo=halo, base=base, kernel=kernel)
        if world > 1:
            tot = res[:1].clone()
            dist.all_reduce(tot)
        return k

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    assert int(res[1].item()) == 0 and int(res[0].item()) == count, "warmup result mismatch"
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    launches = 0
    with ClockSampler(local) as clk:
        t0.record(stream)
        for _ in range(args.steps):
            launches += step()
        t1.record(stream)
        torch.cuda.synchronize()
    ms = t0.elapsed_time(t1) / args.steps
    if world > 1:
        m = torch.tensor([ms], dtype=torch.float64, device=dev)
        dist.all_reduce(m, op=dist.ReduceOp.MAX)
        ms = float(m.item())
        ctot = torch.tensor([count], dtype=torch.int64, device=dev)
        dist.all_reduce(ctot)
        total_count = int(ctot.item())
    else:
        total_count = count
    assert int(res[1].item()) == 0 and int(res[0].item()) == count
    value = world * n * 8 / (ms * 1e-3) / 1e9

    # per-kernel breakdown: the same steps again with events around each launch
    names = ac.last_launch_names()
    nk = len(names)
    pairs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(nk)]
    for a, b in pairs:  # materialise the events
        a.record(stream)
        b.record(stream)
    acc = np.zeros(nk)
    reps = max(3, min(args.steps, 20))
    for _ in range(reps):
        ac.match_async(stt, text, out, res, n_halo=halo, base=base, kernel=kernel, events=pairs)
        torch.cuda.synchronize()
        acc += [a.elapsed_time(b) for a, b in pairs]
    kms = acc / reps
    out_bytes = 8 * count if args.mode == "list" else 0
    # single pass: the scan writes each record to its chain's scratch slot
    # (4 B narrow / 8 B), the gather reads it back and writes the 8-B key
    rec = ac.last_scratch_record_bytes() if args.mode == "list" else 0
    kern = []
    for nm, t in zip(names, kms):
        if "scan" in nm:
            byts = n + (rec * count if "emit1" in nm else out_bytes if "emit" in nm else 0)
        elif "gather" in nm:
            byts = (rec + 8) * count
        else:
            byts = 0  # offset scan / overflow re-walk: latency-bound bookkeeping
        kern.append({"name": nm, "ms": float(t), "share": float(t / ms), "alg_bytes": int(byts)})
    dom = max(kern, key=lambda k: k["ms"])
    hbm, hbm_src, pk = peaks()
    traffic = None
    issue = None
    tf = ROOT / "profiles" / "traffic.json"
    if tf.exists():
        tj = json.loads(tf.read_text())
        traffic = tj.get(f"{args.config}/{args.mode}/{dom['name']}")
        issue = tj.get(f"{args.config}/{args.mode}/{dom['name']}/issue_active")
    achieved = dom["alg_bytes"] / (dom["ms"] * 1e-3) / 1e9
    roof = {"bound": "hbm", "kernel": dom["name"], "achieved": achieved, "peak": hbm, "unit": "GB/s",
            "frac": achieved / hbm, "traffic": traffic, "peak_source": hbm_src,
            # what actually binds this kernel (ncu, same command): the SM issue
            # slots -- fraction of cycles a warp scheduler issued an instruction
            "sm_issue_active_frac": issue,
            "alg_bytes_per_launch": dom["alg_bytes"]}

    line = {
        "metric": METRIC, "value": value, "unit": "Gbps", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u8", "data": "synthetic",
        "config": {"workload": WORKLOADS[args.config], "config": args.config, "mode": args.mode,
                   "bytes_per_gpu": n, "patterns": len(w.patterns), "states": stt.info["n_states"],
                   "classes": stt.info["n_classes"], "stt_bytes": stt.info["stt_bytes"], "tier": stt.tier_name,
                   "kernel": args.kernel, "matches_per_gpu_rank0": count, "matches_total": total_count,
                   "l2": "inputs larger than L2 (256 MiB text + list per step, L2 126 MB)",
                   "parallelism": f"dp{world} (text shards + halo, count all_reduce)"},
        "roofline": roof, "kernels": kern, "gpu_launches": launches,
        "clocks": clk.summary(),
    }

    if not args.no_e2e:
        host = torch.from_numpy(np.ascontiguousarray(text_np[:n])).pin_memory()
        hout = torch.empty(max(1, count + 64), dtype=torch.int64).pin_memory() if args.mode == "list" else None
        c_e2e = ac.match_host(stt, host, hout)
        e_steps = max(3, min(args.steps, 10))
        torch.cuda.synchronize()
        s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s0.record(stream)
        for _ in range(e_steps):
            c_e2e = ac.match_host(stt, host, hout)
        s1.record(stream)
        torch.cuda.synchronize()
        e_ms = s0.elapsed_time(s1) / e_steps
        if world > 1:
            m = torch.tensor([e_ms], dtype=torch.float64, device=dev)
            dist.all_reduce(m, op=dist.ReduceOp.MAX)
            e_ms = float(m.item())
        line["e2e"] = {"value": world * n * 8 / (e_ms * 1e-3) / 1e9, "unit": "Gbps", "h2d_bytes_per_step": n,
                       "d2h_bytes_per_step": 16 + (8 * c_e2e if hout is not None else 0), "steps": e_steps,
                       "ms_per_step": e_ms, "api": "ac_match_host (pinned host text and list)"}
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(w)
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
