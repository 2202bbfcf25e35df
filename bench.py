#!/usr/bin/env python
"""bench.py -- input-text Gbps of the Aho-Corasick matching scan on B200.

One step = one pass of the whole hot path over one
shard of synthetic text: ac_match_async in list mode (single emitting scan
into per-chain scratch slots with the chain offsets computed in its epilogue
-> gather into the canonical list in HBM -> overflow re-walk), plus at N > 1
the combine (all_reduce of the count, allgatherv of the lists).  The STT
build and the host->device copy of the text are outside the timed region, as
in the paper.  The output buffer follows a count-free policy: one
record per 8 text bytes (an output buffer the size of the text), allocated
once before the first scan -- no count pass sizes it.

Workload at N=1: the largest single-GPU configuration of BASELINE.json, C3
(10,000 Snort-like byte patterns over 1 GiB of packet payloads, STT
L1/L2-resident).  C2 and C4 are measured in the same run and reported under
"other_configs".  At N>1 (weak scaling) rank r scans its own 1 GiB segment of
the same C3 text stream plus a (maxlen-1)-byte halo of the next segment;
``--scaling strong --config c4`` splits C4's 4 GiB across the ranks
(plan_shards).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

Prints ONE JSON line (rank 0).  The `--impl reference` arm times the CPU
oracle (oracle/, the only other place this file executes it) on bounded
samples of the same workload on every host core.
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
FALLBACK_HBM_GBS = 7700.0      # B200_PROFILING.md nominal, used only without MEASURED_PEAKS.json
FALLBACK_SM_MHZ = 1965.0
N_SMS = 148
LOOKUPS_PER_SM_CLK = 32        # one conflict-free shared-memory wavefront (32 lanes) per SM per clock


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=50)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", choices=["ours", "reference"], default="ours")
    p.add_argument("--config", default="c3", choices=sorted(WORKLOADS))
    p.add_argument("--scaling", default="weak", choices=["weak", "strong"])
    p.add_argument("--mode", default="list", choices=["list", "count"])
    p.add_argument("--kernel", default="auto", choices=["auto", "staged", "global"])
    p.add_argument("--extra", default="c2,c4", help="other configs measured at N=1 ('' = none)")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-e2e", action="store_true")
    return p.parse_args()


def peaks():
    f = ROOT / "MEASURED_PEAKS.json"
    if f.exists():
        d = json.loads(f.read_text())
        return float(d["hbm_gbs"]), float(d.get("sm_max_mhz", FALLBACK_SM_MHZ)), \
            "measured (MEASURED_PEAKS.json hbm_gbs, sm_max_mhz)"
    return FALLBACK_HBM_GBS, FALLBACK_SM_MHZ, "fallback (B200_PROFILING.md)"


def bench_config(args, world: int) -> dict:
    """The `config` object, identical in both arms for the same arguments."""
    if args.scaling == "strong":
        par = f"dp{world} strong: one text split in {world} shards + halo"
    else:
        par = f"dp{world} weak: one text segment per rank + halo"
    return {"workload": WORKLOADS[args.config], "config": args.config, "mode": args.mode,
            "scaling": args.scaling, "parallelism": par,
            "combine": "all_reduce(count) + allgatherv(lists)" if world > 1 else "none",
            "out_capacity": "n/8 records per shard, count-free",
            "l2": "inputs larger than L2 (text >= 256 MiB per step, L2 126 MB): no flush"}


def all_reduce(t, op=None):
    """all_reduce in place; through host memory when the group is gloo (the
    functional check of the N > 1 path), on the device over NCCL otherwise."""
    import torch.distributed as dist
    op = op if op is not None else dist.ReduceOp.SUM
    if dist.get_backend() == "gloo" and t.is_cuda:
        h = t.cpu()
        dist.all_reduce(h, op=op)
        t.copy_(h)
    else:
        dist.all_reduce(t, op=op)
    return t


def cpu_model() -> str:
    try:
        for line in Path("/proc/cpuinfo").read_text().splitlines():
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


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
            time.sleep(0.002)

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
def load_workload(cfg: str, rank: int, world: int = 1, scaling: str = "weak"):
    """Returns (workload, this rank's bytes, owned bytes, halo, base)."""
    import synth
    t0 = time.time()
    w = synth.make(cfg)
    maxlen = max(len(p) for p in w.patterns)
    if scaling == "strong" and world > 1:
        from paper_conf_ipps_tranlhc13_b200.dist import plan_shards
        sh = plan_shards(w.text.size, world, maxlen)[rank]
        text, owned, halo, base = w.text[sh.lo:sh.read_hi], sh.owned, sh.halo, sh.lo
    else:
        halo = maxlen - 1 if world > 1 else 0
        owned = w.text.size
        base = rank * owned
        if rank == 0:
            text = w.text
            if halo:
                text = np.concatenate([w.text, synth.stream(w, cfg, w.text.size // synth.BLOCK, halo)])
        else:
            text = synth.segment(w, cfg, rank, w.text.size, halo)
    log(f"[rank {rank}] workload {cfg}: {owned} B owned (+{halo} halo), {len(w.patterns)} patterns, "
        f"gen {time.time() - t0:.1f}s")
    return w, np.ascontiguousarray(text), owned, halo, base


# ----------------------------------------------------- the oracle on the host
def oracle_rate(w, text, seconds: float, threads: int):
    """The oracle as it stands, timed on `threads` host cores over a sample of
    `text` sized for about `seconds` of work: (Gbps, sample bytes, wall s,
    matches).  Canonical lists, build excluded."""
    from oracle import Oracle
    o = Oracle(w.patterns)
    probe = min(text.size, 1 << 20)
    t0 = time.perf_counter()
    o.match(text[:probe])
    rate = probe / max(1e-6, time.perf_counter() - t0) * threads
    size = int(min(text.size, max(probe, rate * seconds)))
    t0 = time.perf_counter()
    if threads == 1:
        ends, _ = o.match(text[:size])
    else:
        ends, _ = o.match_parallel(text[:size], threads=threads)
    dt = time.perf_counter() - t0
    return size * 8 / dt / 1e9, size, dt, int(ends.size)


def cpu_baseline(w, text, cfg):
    cores = os.cpu_count() or 1
    v, size, dt, _ = oracle_rate(w, text, 10.0, cores)
    v1, size1, dt1, _ = oracle_rate(w, text, 4.0, 1)
    return {"value": v, "unit": "Gbps", "cores": cores, "kind": "oracle", "cpu_model": cpu_model(),
            "sample": f"first {size} B of the {cfg} text as {cores} start-owned windows on {cores} threads "
                      f"(canonical list), build excluded, {dt:.1f} s",
            "single_thread": {"value": v1, "unit": "Gbps", "cores": 1,
                              "sample": f"first {size1} B, 1 thread, {dt1:.1f} s"}}


# ------------------------------------------------------------ reference arm
def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", str(args.gpus)))
    if rank != 0:
        return 0
    from oracle import Oracle
    w, text, owned, _, _ = load_workload(args.config, 0)
    n = owned
    cores = os.cpu_count() or 1
    o = Oracle(w.patterns)
    probe = min(n, 1 << 20)
    t0 = time.perf_counter()
    o.match(text[:probe])
    rate = probe / max(1e-6, time.perf_counter() - t0) * cores
    per_step = int(min(n, max(1 << 16, rate * 100.0 / max(1, args.steps + args.warmup))))
    rng = np.random.default_rng(0)
    los = rng.integers(0, max(1, n - per_step), size=args.steps + args.warmup)
    tot_b, tot_t, cnt = 0, 0.0, 0
    for i, lo in enumerate(los):
        t0 = time.perf_counter()
        ends, _ = o.match_parallel(text[lo:lo + per_step], threads=cores)
        dt = time.perf_counter() - t0
        if i >= args.warmup:
            tot_b += per_step
            tot_t += dt
            cnt += ends.size
    gbps = tot_b * 8 / tot_t / 1e9
    sample = (f"{args.steps} windows of {per_step} B at seeded offsets of the {args.config} text, each as {cores} "
              f"start-owned sub-windows on {cores} threads (canonical list), build excluded")
    line = {
        "impl": "reference", "metric": METRIC, "value": gbps, "unit": "Gbps", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": tot_t / args.steps * 1e3,
        "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None, "dtype": "u8", "data": "synthetic",
        "config": bench_config(args, world),
        "cpu_baseline": {"value": gbps, "unit": "Gbps", "cores": cores, "kind": "oracle", "cpu_model": cpu_model(),
                         "sample": sample},
        "e2e": {"value": gbps, "unit": "Gbps", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "sample_bytes_per_step": per_step, "matches_in_sample": int(cnt),
    }
    print(json.dumps(line), flush=True)
    return 0


# ---------------------------------------------------------------- our arm
def time_config(args, cfg: str, rank: int, world: int, dev, local: int, steps: int, warmup: int,
                clocks: bool, e2e: bool):
    """Build, warm up and time one configuration; returns (line fields, w, text)."""
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_tranlhc13_b200 as ac
    from paper_conf_ipps_tranlhc13_b200.dist import allgatherv, default_capacity

    w, text_np, owned, halo, base = load_workload(cfg, rank, world, args.scaling)
    stt = ac.build(w.patterns, device=local)
    text = torch.from_numpy(text_np).to(dev)
    kernel = {"auto": ac.KERNEL_AUTO, "staged": ac.KERNEL_STAGED, "global": ac.KERNEL_GLOBAL}[args.kernel]
    res = torch.zeros(2, dtype=torch.int64, device=dev)
    out = torch.empty(default_capacity(owned), dtype=torch.int64, device=dev) if args.mode == "list" else None
    stream = torch.cuda.current_stream()

    def step():
        k = ac.match_async(stt, text, out, res, n_halo=halo, base=base, kernel=kernel)
        if world > 1:
            tot = res[:1].clone()
            all_reduce(tot)
            if out is not None:
                allgatherv(out[:int(res[0].item())])
        return k

    for _ in range(warmup):
        step()
    torch.cuda.synchronize()
    count, status = (int(x) for x in res.tolist())
    assert status == 0, f"{cfg}: status {status} (count {count}) -- output capacity policy too small"
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    launches = 0
    clk = ClockSampler(local) if clocks else None
    if clk:
        clk.__enter__()
    t0.record(stream)
    for _ in range(steps):
        launches += step()
    t1.record(stream)
    torch.cuda.synchronize()
    if clk:
        clk.__exit__()
    ms = t0.elapsed_time(t1) / steps
    total_owned = owned
    if world > 1:
        m = torch.tensor([ms], dtype=torch.float64, device=dev)
        all_reduce(m, op=dist.ReduceOp.MAX)
        ms = float(m.item())
        agg = torch.tensor([count, owned], dtype=torch.int64, device=dev)
        all_reduce(agg)
        total_count, total_owned = (int(x) for x in agg.tolist())
    else:
        total_count = count
    assert int(res[1].item()) == 0 and int(res[0].item()) == count
    value = total_owned * 8 / (ms * 1e-3) / 1e9

    # per-kernel breakdown: the same scan again with events around each launch
    # (recorded on the stream each kernel runs on; head/tail chains run on a
    # side stream, overlapped with the main scan)
    names = ac.last_launch_names()
    nk = len(names)
    pairs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(nk)]
    for a, b in pairs:
        a.record(stream)
        b.record(stream)
    acc = np.zeros(nk)
    reps = max(3, min(steps, 20))
    for _ in range(reps):
        ac.match_async(stt, text, out, res, n_halo=halo, base=base, kernel=kernel, events=pairs)
        torch.cuda.synchronize()
        acc += [a.elapsed_time(b) for a, b in pairs]
    tbytes = ac.last_launch_text_bytes()
    kms = acc / reps
    staged = any("scan_staged" in x for x in names)  # head/tail chains then run on the side stream
    kern = []
    for nm, t, tb in zip(names, kms, tbytes):
        # SURVEY 8(d) algorithmic bytes: text read by the scans, final 8-byte
        # records written by the gather (scratch records are intermediates)
        alg = tb if "scan" in nm else 8 * count if "gather" in nm else 0
        kern.append({"name": nm, "ms": float(t), "share": float(t / ms), "text_bytes": int(tb),
                     "alg_bytes": int(alg), "stream": "side (overlapped)" if "scan_global" in nm and staged else "main"})
    main = [k for k in kern if k["stream"] == "main"]
    dom = max(main, key=lambda k: k["ms"])
    hbm, sm_mhz, src = peaks()
    tf = ROOT / "profiles" / "traffic.json"
    tj = json.loads(tf.read_text()) if tf.exists() else {}
    key = f"{cfg}/{args.mode}/{dom['name']}"
    traffic = tj.get(key)
    unit_note = tj.get(f"{key}/binding")
    lookups = dom["text_bytes"]  # one STT transition per owned text byte
    achieved = lookups / (dom["ms"] * 1e-3) / 1e9
    peak_lk = N_SMS * sm_mhz * 1e6 * LOOKUPS_PER_SM_CLK / 1e9
    step_alg = owned + 8 * count
    roof = {"bound": "alu", "kernel": dom["name"], "achieved": achieved, "peak": peak_lk, "unit": "Glookup/s",
            "frac": achieved / peak_lk, "traffic": traffic,
            "peak_source": f"{N_SMS} SMs x {sm_mhz:.0f} MHz x {LOOKUPS_PER_SM_CLK} lookups (one conflict-free "
                           f"shared-memory wavefront per SM-clock; DESIGN.md section 7); {src}",
            "binding_unit_ncu": unit_note,
            "hbm": {"achieved": dom["alg_bytes"] / (dom["ms"] * 1e-3) / 1e9, "peak": hbm, "unit": "GB/s",
                    "frac": dom["alg_bytes"] / (dom["ms"] * 1e-3) / 1e9 / hbm,
                    "alg_bytes_per_launch": dom["alg_bytes"],
                    "step_alg_bytes": step_alg, "step_frac": step_alg / (ms * 1e-3) / 1e9 / hbm}}
    fields = {"value": value, "ms_per_step": ms, "roofline": roof, "kernels": kern, "gpu_launches": launches,
              "workload_info": {"bytes_per_gpu": owned, "patterns": len(w.patterns), "states": stt.info["n_states"],
                                "classes": stt.info["n_classes"], "stt_bytes": stt.info["stt_bytes"],
                                "tier": stt.tier_name, "kernel": args.kernel, "matches_rank0": count,
                                "matches_total": total_count}}
    if clk:
        fields["clocks"] = clk.summary()
    if e2e:
        host = torch.from_numpy(np.ascontiguousarray(text_np[:owned])).pin_memory()
        hout = torch.empty(default_capacity(owned), dtype=torch.int64).pin_memory() if args.mode == "list" else None
        c_e2e = ac.match_host(stt, host, hout)
        e_steps = max(3, min(steps, 10))
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
            all_reduce(m, op=dist.ReduceOp.MAX)
            e_ms = float(m.item())
        fields["e2e"] = {"value": total_owned * 8 / (e_ms * 1e-3) / 1e9, "unit": "Gbps", "h2d_bytes_per_step": owned,
                         "d2h_bytes_per_step": 16 + (8 * c_e2e if hout is not None else 0), "steps": e_steps,
                         "ms_per_step": e_ms, "api": "ac_match_host (pinned host text and list)"}
        del host, hout
    del text, out
    torch.cuda.empty_cache()
    return fields, w, text_np[:owned]


def run_ours(args):
    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # AC_BENCH_BACKEND=gloo: a functional check of the N > 1 path on a box
    # with fewer GPUs than ranks (ranks share devices, collectives go through
    # host memory); the contract run uses NCCL, one GPU per rank
    backend = os.environ.get("AC_BENCH_BACKEND", "nccl")
    if backend != "nccl":
        local = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    dev = torch.device("cuda", local)
    fields, w, text_np = time_config(args, args.config, rank, world, dev, local, args.steps, args.warmup, True,
                                     not args.no_e2e)
    line = {"metric": METRIC, "value": fields.pop("value"), "unit": "Gbps", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": fields.pop("ms_per_step"), "higher_is_better": True,
            "scaling": args.scaling, "vs_baseline": None, "dtype": "u8", "data": "synthetic",
            "config": bench_config(args, world)}
    line.update(fields)
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(w, text_np, args.config)
    del w, text_np
    if world == 1 and args.extra:
        other = {}
        for cfg in [c for c in args.extra.split(",") if c and c != args.config]:
            f, _, _ = time_config(args, cfg, 0, 1, dev, local, max(3, min(args.steps, 20)), 3, False, False)
            other[cfg] = {"workload": WORKLOADS[cfg], "value": f["value"], "unit": "Gbps",
                          "ms_per_step": f["ms_per_step"], "roofline_frac": f["roofline"]["frac"],
                          "hbm_frac": f["roofline"]["hbm"]["frac"], "dominant": f["roofline"]["kernel"],
                          "workload_info": f["workload_info"], "kernels": f["kernels"]}
        line["other_configs"] = other
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
