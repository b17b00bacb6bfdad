#!/usr/bin/env python
"""Benchmark of the B200 ARBALEST replay (BASELINE.json metric: events/sec replayed
at 1/2/4/8 B200 and % of HBM roofline; vs CPU oracle).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload config5|config3|config4|config2]
    python -m torch.distributed.run --nproc-per-node N --master-addr 127.0.0.1 ... bench.py --gpus N
    python bench.py --impl reference ...     (the CPU oracle, timed on the host cores)

One step = one pass of the whole hot path (decode + partition, control
resolution, replay + classification, MIR join, report compaction, count
exchange) over the whole named workload.  Default: config 5, the 9.0e9-record
trace over 2^33 words (64 GiB of locations) -- strong scaling: rank r of N owns
the words [r * 2^33 / N, (r + 1) * 2^33 / N) and replays every record touching
them (all control records replicated).  The trace is cut into 9
time batches at quiescent points ("1-GPU = the same total trace,
in quiescent batches"; 9 so that each batch is one flush of <= 2^30 records,
the ABI's maximum); each batch is generated on the device (untimed) and its
flushes are timed with CUDA events on the replay stream between a barrier + a
synchronize; a step's time is the sum over batches of the max over ranks.
Events = word-events: one per (tracked word, data op).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "events/sec replayed (1/2/4/8 B200) and % of HBM roofline; vs CPU oracle"
UNIT = "word-events/s"
MAX_FLUSH = 1 << 30          # records per flush: the ABI's maximum batch (arb_submit_events)
DEFAULT_BATCHES = 9          # config 5: 9 quiescent time batches of ~1.0e9 records -> one flush each


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as fh:
            d = json.load(fh)
        return float(d["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


def host_info():
    info = {"nproc": os.cpu_count()}
    try:
        info["nproc"] = int(subprocess.check_output(["nproc"], text=True).strip())
        info["free_g"] = subprocess.check_output(["free", "-g"], text=True).strip().splitlines()[1]
    except Exception:
        pass
    return info


class ClockSampler:
    """nvidia-smi clocks/throttle reasons sampled during the timed region."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device):
        self.device = device
        self.p = None

    def start(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--id={self.device}", f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "100"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.p = None

    def stop(self):
        if not self.p:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        out, _ = self.p.communicate(timeout=10)
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx = float(f[2])
            except ValueError:
                continue
            for n, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(n)
        load = [x for x in sm if mx and x > 0.5 * mx] or sm
        return {"sm_mhz": float(np.median(load)) if load else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


# ---------------------------------------------------------------------------
# workloads
# ---------------------------------------------------------------------------
def make_program(name, scale=1.0):
    from gen import native
    if name == "config5":
        return native.config5(total_records=int(9e9 * scale))
    if name == "config3":
        return native.config3(scale=scale)
    if name == "config4":
        return native.config4(scale=scale)
    if name == "config2":
        return native.from_records("config2", *__import__("gen.configs", fromlist=["config2"]).config2())
    raise SystemExit(f"unknown workload {name}")


def word_space(prog):
    from gen import native
    if prog.name == "config5":
        return native.C5_BASE_WORD, native.C5_WORDS
    return prog.addr_base // 8, prog.addr_bytes // 8


def rank_range(prog, rank, world):
    from paper_conf_ipps_yuphs21_b200.shard import shard_range
    base, n = word_space(prog)
    return shard_range(base, n, rank, world)


def time_batches(prog, n_batches):
    """Global record ranges [g0, g1) cut at quiescent points into ~n_batches pieces."""
    q = np.asarray(prog.quiescent, dtype=np.int64)
    cuts = [0]
    for k in range(1, n_batches):
        target = prog.n * k // n_batches
        c = int(q[np.searchsorted(q, target)]) if target <= q[-1] else prog.n
        if c > cuts[-1] and c < prog.n:
            cuts.append(c)
    cuts.append(prog.n)
    return [(a, b) for a, b in zip(cuts[:-1], cuts[1:]) if b > a]


class BatchSource:
    """Generates the records of global batch [g0, g1) that touch words [lo, hi) on the
    device (all records when [lo, hi) is the program's whole word space, else every
    control record + the accesses touching the range, with global indices), and cuts
    them into flushes at quiescent points."""

    def __init__(self, prog, lo, hi, device, chunk=1 << 27):
        import torch
        self.prog, self.lo, self.hi, self.device, self.chunk = prog, lo, hi, device, chunk
        base, n = word_space(prog)
        self.whole = (lo, hi) == (base, base + n)
        self.tmp = None if self.whole else torch.empty((chunk, 2), dtype=torch.int64, device=device)
        self.buf = None
        self.gbuf = None

    def _grow(self, cap, keep):
        import torch
        nb = torch.empty((cap, 2), dtype=torch.int64, device=self.device)
        ng = torch.empty(cap, dtype=torch.int64, device=self.device)
        if keep:
            nb[:keep].copy_(self.buf[:keep])
            ng[:keep].copy_(self.gbuf[:keep])
        self.buf, self.gbuf = nb, ng

    def make(self, g0, g1):
        import torch
        from gen import native
        n = g1 - g0
        if self.whole:
            if self.buf is None or self.buf.shape[0] < n:
                self.buf = None
                torch.cuda.empty_cache()
                self.buf = torch.empty((n, 2), dtype=torch.int64, device=self.device)
            self.prog.fill_device(self.buf, g0, n)
            recs, gidx, k = self.buf[:n], None, n
        else:
            # capacity: the rank's share of the batch plus one chunk (grown if exceeded)
            base, nw = word_space(self.prog)
            want = int(n * (self.hi - self.lo) / nw * 1.25) + self.chunk
            if self.buf is None or self.buf.shape[0] < min(want, n + 1):
                self._grow(min(want, n + 1), 0)
            k = 0
            s = g0
            while s < g1:
                cnt = min(self.chunk, g1 - s)
                if self.buf.shape[0] - k < cnt:
                    self._grow(k + cnt + self.chunk * 4, k)
                self.prog.fill_device(self.tmp, s, cnt)
                k += native.filter_device(self.tmp, cnt, self.lo, self.hi, s, self.buf[k:], self.gbuf[k:])
                s += cnt
            recs, gidx = self.buf[:k], self.gbuf[:k]
        # flush cuts: local positions of the quiescent global indices inside the batch
        q = np.asarray(self.prog.quiescent, dtype=np.int64)
        q = q[(q > g0) & (q < g1)]
        if gidx is None:
            local_q = (q - g0).tolist()
        else:
            local_q = torch.searchsorted(gidx, torch.tensor(q, device=self.device)).cpu().numpy().tolist()
        # as few flushes as the 2^30-record limit allows, cut near equal sizes
        nf = max(1, -(-k // MAX_FLUSH))
        cuts = [0]
        qa = np.asarray(local_q, dtype=np.int64)
        for j in range(1, nf):
            want = k * j // nf
            ok = qa[(qa > cuts[-1]) & (qa - cuts[-1] <= MAX_FLUSH)]
            if ok.size:
                cuts.append(int(ok[np.argmin(np.abs(ok - want))]))
        if cuts[-1] != k:
            cuts.append(k)
        assert all(b - a <= MAX_FLUSH for a, b in zip(cuts[:-1], cuts[1:])), "no quiescent cut below 2^30 records"
        flushes = [(a, b) for a, b in zip(cuts[:-1], cuts[1:]) if b > a] or [(0, 0)]
        return recs, gidx, flushes


STAT_KEYS = ("access_words", "range_words", "reports", "records", "ms_partition", "ms_replay", "ms_mir",
             "ms_reports", "ms_control", "ms_total", "ms_sample", "ms_segsort", "ms_host_control", "steps_fast",
             "steps_sort", "steps_run", "segments", "chunks", "chunks_fast", "chunks_run", "run_merges", "work_items", "hot_buckets", "kernel_launches", "exchanges")


def run_workload(prog, ctx, src, batches, steps, warmup, stream, world, dev, on_batch=None, clocks=None):
    """Warm-up + timed steps over all batches; returns (per-step ms (job), per-step stats of the
    last step, per-batch info).  Per batch: generate (untimed), equalise the flush count
    across ranks, barrier + synchronize, CUDA events around the flushes, synchronize."""
    import torch
    import torch.distributed as dist
    step_ms = []
    last = None
    info = []
    for it in range(warmup + steps):
        timed = it >= warmup
        if timed and clocks is not None and it == warmup:
            clocks.start()
        acc = {k: 0 for k in STAT_KEYS}
        acc["by_kind"] = [0, 0, 0, 0]
        acc["max_bucket_events"] = 0
        acc["flushes"] = 0
        t_step = 0.0
        for bi, (g0, g1) in enumerate(batches):
            recs, gidx, flushes = src.make(g0, g1)
            if world > 1:
                nf = torch.tensor([len(flushes)], dtype=torch.int64, device=dev)
                dist.all_reduce(nf, op=dist.ReduceOp.MAX)
                flushes = flushes + [(flushes[-1][1], flushes[-1][1])] * (int(nf.item()) - len(flushes))
            torch.cuda.synchronize()
            if world > 1:
                dist.barrier()
            ev0 = torch.cuda.Event(enable_timing=True)
            ev1 = torch.cuda.Event(enable_timing=True)
            ev0.record(stream)
            for (a, b) in flushes:
                if b > a:
                    ctx.submit_events(recs[a:b], global_index=None if gidx is None else gidx[a:b], stream=stream)
                rc, n, off = ctx.flush(stream=stream)
                st = ctx.stats()
                for k in STAT_KEYS:
                    acc[k] += st[k]
                acc["max_bucket_events"] = max(acc["max_bucket_events"], st["max_bucket_events"])
                acc["flushes"] += 1 if b > a else 0
                for k in range(4):
                    acc["by_kind"][k] += st["reports_by_kind"][k]
            ev1.record(stream)
            torch.cuda.synchronize()
            ms = ev0.elapsed_time(ev1)
            t = torch.tensor([ms], dtype=torch.float64, device=dev)
            if world > 1:
                dist.all_reduce(t, op=dist.ReduceOp.MAX)
            t_step += float(t.item())
            if on_batch is not None and it == warmup:
                on_batch(bi, recs, gidx, flushes)
            if it == 0:
                info.append({"global": [g0, g1], "records": int(recs.shape[0]), "flushes": len(flushes)})
        if timed:
            step_ms.append(t_step)
            last = acc
    return step_ms, last, info


def run_reference(args):
    """--impl reference: the CPU oracle as it stands, on the host cores, on a bounded
    sample of the same workload (rank 0 only)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    prog = make_program(args.workload, args.scale)
    lo, hi = rank_range(prog, 0, 1)
    rec = prog.fill_host(0, min(prog.n, args.ref_sample))
    cut = quiescent_prefix(prog, np.arange(rec.shape[0]), args.ref_sample)
    rec = rec[:cut]
    threads = os.cpu_count() or 1
    times, evs = [], 0
    for s in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        r = oracle.replay(rec, lo * 8, (hi - lo) * 8, want_shadow=False, threads=threads)
        dt = time.perf_counter() - t0
        assert r.rc == 0
        if s >= args.warmup:
            times.append(dt)
            evs = r.stats["word_events"]
    v = evs / float(np.mean(times))
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * float(np.mean(times)),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u8",
            "data": "synthetic",
            "config": {"workload": args.workload, "sample_records": int(rec.shape[0]),
                       "sample_word_events": int(evs), "host": host_info()},
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": threads, "kind": "oracle",
                             "sample": f"first {rec.shape[0]} records of {args.workload} (whole word space), "
                                       f"address-sharded over {threads} threads"},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def quiescent_prefix(prog, gidx, budget):
    """Largest prefix of a rank's records (global indices gidx, ascending) that ends
    at a quiescent point of the program and holds <= budget records (else the
    shortest non-empty one): a bounded sample never cuts a nowait block open."""
    q = np.asarray(prog.quiescent, dtype=np.int64)
    local = np.unique(np.searchsorted(np.asarray(gidx, dtype=np.int64), q))
    local = local[local > 0]
    if local.size == 0:
        return len(gidx)
    ok = local[local <= budget]
    return int(ok[-1]) if ok.size else int(local[0])


def cpu_baseline(prog, recs_dev, gidx_dev, lo, hi, budget_records, g0):
    """The oracle as it stands on a bounded sample of the first batch: single-threaded
    and address-sharded over all host cores."""
    import oracle
    gi_all = (np.arange(recs_dev.shape[0], dtype=np.int64) + g0) if gidx_dev is None else gidx_dev.cpu().numpy()
    n = quiescent_prefix(prog, gi_all, min(budget_records, recs_dev.shape[0]))
    rec = recs_dev[:n].cpu().numpy().view(np.uint64)
    gi = gi_all[:n].view(np.uint64) if gidx_dev is not None else None
    out = {}
    cores = os.cpu_count() or 1
    for label, th in (("1core", 1), ("all_cores", cores)):
        t0 = time.perf_counter()
        r = oracle.replay(rec, lo * 8, (hi - lo) * 8, global_index=gi, want_shadow=False, threads=th)
        dt = time.perf_counter() - t0
        assert r.rc == 0, r.rc
        out[label] = {"value": r.stats["word_events"] / dt, "threads": th, "s": round(dt, 2),
                      "word_events": r.stats["word_events"]}
    hi_v = out["all_cores"]
    return {"value": hi_v["value"], "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"first {n} records of the first batch ({hi_v['word_events']} word-events); "
                      f"plain C, address-sharded over {cores} threads ({hi_v['s']} s); "
                      f"single-threaded: {out['1core']['value']:.3g} word-events/s ({out['1core']['s']} s)",
            "single_core": out["1core"]["value"], "host": host_info()}


def roofline(prog, s0, lo, hi, batches, ms_per_step, hbm_gbs, peak_src, n_busy):
    """B_alg = 16 R + 2 W + 16 Rep per flush; per-kernel algorithmic bytes
     over the kernel's CUDA-event time."""
    # W per flush ~ W per batch (the sections entered in the batch, clipped to [lo, hi))
    W = sum(prog.distinct_words(lo, hi, batches))
    W_sec = sum(prog.distinct_words(lo, hi, batches, sector_words=32))
    b_alg = 16 * s0["records"] + 2 * W + 16 * s0["reports"]
    b_alg_sec = 16 * s0["records"] + 2 * W_sec + 16 * s0["reports"]
    phases = {"k_sample+balance": s0["ms_sample"], "k_partition": s0["ms_partition"] - s0["ms_sample"],
              "k_replay": s0["ms_replay"], "k_mir": s0["ms_mir"],
              "report_compaction": s0["ms_reports"], "control_plane": s0["ms_control"],
              "segment_sort (in control_plane)": s0["ms_segsort"],
              "host_control_wall (in control_plane)": s0["ms_host_control"]}
    alg = {"k_partition": 16 * s0["records"], "k_replay": 2 * W + 16 * s0["reports"]}
    dom = max(("k_partition", "k_replay"), key=lambda k: phases[k])
    achieved = alg[dom] / (phases[dom] / 1e3) / 1e9 if phases[dom] > 0 else 0.0
    traffic = None
    kern = {}
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as fh:
            tj = json.load(fh)
    except Exception:
        tj = {}
    for k in ("k_partition", "k_replay"):
        ach = alg[k] / (phases[k] / 1e3) / 1e9 if phases[k] > 0 else 0.0
        kern[k] = {"ms_per_step": phases[k], "alg_bytes_per_step": alg[k], "achieved": ach, "frac": ach / hbm_gbs}
        if k in tj:
            kern[k]["ncu_dram_bytes_per_record"] = tj[k]["dram_bytes_per_launch"] / tj[k]["records_in_launch"]
    if dom in tj:
        traffic = tj[dom]["dram_bytes_per_launch"] / tj[dom]["records_in_launch"] * s0["records"] / n_busy
    path_ach = b_alg / (ms_per_step / 1e3) / 1e9
    roof = {"bound": "hbm", "kernel": dom, "achieved": achieved, "peak": hbm_gbs, "unit": "GB/s",
            "frac": achieved / hbm_gbs, "traffic": traffic, "traffic_unit": "bytes per launch (ncu)",
            "alg_bytes_per_launch": alg[dom] / n_busy, "peak_source": peak_src,
            "kernel_ms_per_step": phases[dom], "phase_ms_per_step": phases, "kernels": kern,
            "path": {"b_alg_bytes_per_step": b_alg, "W": W, "achieved": path_ach, "frac": path_ach / hbm_gbs,
                     "sector_granular": {"W_sectors_x32": W_sec, "b_alg_bytes_per_step": b_alg_sec,
                                         "frac": b_alg_sec / (ms_per_step / 1e3) / 1e9 / hbm_gbs}}}
    if dom == "k_replay":
        roof["note"] = ("k_replay's algorithmic bytes are the shadow (2 B per distinct word) and the reports "
                        "(16 B each), SURVEY §8(d); the partition events it reads are design overhead, so its HBM "
                        "fraction is small by construction; kernels.k_partition (reads the trace, 16 B/record) and "
                        "path (B_alg / step time) carry the HBM roofline")
    return roof


def side_workload(name, args, dev, stream, world, rank, hbm_gbs, peak_src, flags):
    """configs 3 / 4 (one batch each) at the same rank layout: value and roofline."""
    from paper_conf_ipps_yuphs21_b200 import Context
    prog = make_program(name, 1.0)
    lo, hi = rank_range(prog, rank, world)
    src = BatchSource(prog, lo, hi, dev)
    batches = time_batches(prog, 1)
    ctx = Context(lo * 8, (hi - lo) * 8, device=dev.index, flags=flags, report_capacity=1 << 25)
    ms, s0, info = run_workload(prog, ctx, src, batches, args.side_steps, 2, stream, world, dev)
    ctx.close()
    del src
    ms_step = float(np.mean(ms))
    import torch
    import torch.distributed as dist
    tot = torch.tensor([s0["access_words"] + s0["range_words"], s0["access_words"]], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(tot)
    roof = roofline(prog, s0, lo, hi, batches, ms_step, hbm_gbs, peak_src, max(1, s0["flushes"]))
    return {"value": float(tot[0]) / (ms_step / 1e3), "unit": UNIT, "ms_per_step": ms_step,
            "access_word_events_per_s": float(tot[1]) / (ms_step / 1e3),
            "records_per_step_rank0": int(s0["records"]), "word_events_per_step": int(tot[0]),
            "reports_rank0": int(s0["reports"]), "flushes_rank0": int(s0["flushes"]),
            "path_frac": roof["path"]["frac"], "dominant": roof["kernel"], "dominant_frac": roof["frac"],
            "phase_ms_per_step": roof["phase_ms_per_step"], "steps": args.side_steps, "warmup": 2}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="config5")
    ap.add_argument("--scale", type=float, default=1.0)
    ap.add_argument("--batches", type=int, default=DEFAULT_BATCHES, help="time batches of the trace (quiescent cuts)")
    ap.add_argument("--max-batches", type=int, default=0, help="profiling: replay only the first K batches")
    ap.add_argument("--e2e-steps", type=int, default=1)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-side", action="store_true", help="skip the config 3 / 4 side measurements")
    ap.add_argument("--side-steps", type=int, default=3)
    ap.add_argument("--dedup", action="store_true", help="ARB_F_DEDUP_FIRST reporting (the production mode; with "
                                                        "repeated steps on one context its set persists, so later "
                                                        "steps find no new pairs) instead of raw reporting")
    ap.add_argument("--bo", action="store_true", help="enable the buffer-overflow extension (ARB_F_BO, Z20)")
    ap.add_argument("--cpu-records", type=int, default=200_000_000)
    ap.add_argument("--ref-sample", type=int, default=30_000_000)
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist
    from paper_conf_ipps_yuphs21_b200 import Context, ARB_F_TIMING, ARB_F_BO, ARB_F_DEDUP_FIRST
    from paper_conf_ipps_yuphs21_b200.shard import nccl_unique_id

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    hbm_gbs, peak_src = peaks()
    flags = ARB_F_TIMING | (ARB_F_BO if args.bo else 0) | (ARB_F_DEDUP_FIRST if args.dedup else 0)

    prog = make_program(args.workload, args.scale)
    lo, hi = rank_range(prog, rank, world)
    batches = time_batches(prog, args.batches if prog.name == "config5" else 1)
    if args.max_batches:
        batches = batches[:args.max_batches]
    src = BatchSource(prog, lo, hi, dev)

    uid = None
    if world > 1:
        buf = torch.zeros(128, dtype=torch.uint8, device=dev)
        if rank == 0:
            buf.copy_(torch.frombuffer(bytearray(nccl_unique_id()), dtype=torch.uint8))
        dist.broadcast(buf, 0)
        uid = bytes(buf.cpu().numpy().tobytes())
    ctx = Context(lo * 8, (hi - lo) * 8, device=local, rank=rank, world=world, nccl_unique_id=uid,
                  flags=flags, report_capacity=1 << 25)
    stream = torch.cuda.Stream(device=dev)

    cpu_state = {}

    def keep_first(bi, recs, gidx, flushes):      # the oracle baseline samples the first batch
        if bi == 0 and rank == 0 and world == 1 and not args.no_cpu:
            n = min(args.cpu_records, recs.shape[0])
            cpu_state["recs"] = recs[:n].clone()
            cpu_state["gidx"] = None if gidx is None else gidx[:n].clone()

    clocks = ClockSampler(local)
    t_wall = time.perf_counter()
    ms_steps, s0, binfo = run_workload(prog, ctx, src, batches, args.steps, args.warmup, stream, world, dev,
                                       on_batch=keep_first, clocks=clocks)
    clk = clocks.stop()
    t_wall = time.perf_counter() - t_wall
    ms_per_step = float(np.mean(ms_steps))
    tot = torch.tensor([s0["access_words"] + s0["range_words"], s0["records"], s0["reports"], s0["access_words"],
                        s0["kernel_launches"]], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(tot)
    word_events_all, records_all, reports_all, access_all, launches_all = [float(x) for x in tot.tolist()]
    value = word_events_all / (ms_per_step / 1e3)
    roof = roofline(prog, s0, lo, hi, batches, ms_per_step, hbm_gbs, peak_src, max(1, s0["flushes"]))

    # ---- e2e: host buffers through the public API, per batch ------------------------
    e2e = None
    if not args.no_e2e:
        t_e2e, h2d, d2h = 0.0, 0, 0
        hbuf = None
        for _ in range(args.e2e_steps):
            for (g0, g1) in batches:
                recs, gidx, flushes = src.make(g0, g1)
                if world > 1:
                    nf = torch.tensor([len(flushes)], dtype=torch.int64, device=dev)
                    dist.all_reduce(nf, op=dist.ReduceOp.MAX)
                    flushes = flushes + [(flushes[-1][1], flushes[-1][1])] * (int(nf.item()) - len(flushes))
                if hbuf is None or hbuf.shape[0] < recs.shape[0]:
                    hbuf = torch.empty((recs.shape[0], 2), dtype=torch.int64, pin_memory=True)
                    hg = torch.empty(recs.shape[0], dtype=torch.int64, pin_memory=True) if gidx is not None else None
                h_rec = hbuf[:recs.shape[0]]
                h_rec.copy_(recs)
                h_gi = None
                if gidx is not None:
                    h_gi = hg[:recs.shape[0]]
                    h_gi.copy_(gidx)
                torch.cuda.synchronize()
                if world > 1:
                    dist.barrier()
                t0 = time.perf_counter()
                for (a, b) in flushes:
                    if b > a:
                        ctx.submit_events(h_rec[a:b], global_index=None if h_gi is None else h_gi[a:b],
                                          stream=stream)
                    rc, n, off = ctx.flush(stream=stream)
                    rep = ctx.get_reports(n)
                    d2h += rep.nbytes + 16
                torch.cuda.synchronize()
                dt = torch.tensor([time.perf_counter() - t0], dtype=torch.float64, device=dev)
                if world > 1:
                    dist.all_reduce(dt, op=dist.ReduceOp.MAX)
                t_e2e += float(dt.item())
                h2d += int(recs.numel() * 8 + (0 if gidx is None else gidx.numel() * 8))
        del hbuf
        e2e = {"value": word_events_all * args.e2e_steps / t_e2e, "unit": UNIT,
               "h2d_bytes_per_step": h2d // args.e2e_steps, "d2h_bytes_per_step": d2h // args.e2e_steps,
               "note": "per batch: pinned host records -> arb_submit_events (host pointer) -> arb_flush -> "
                       "arb_get_reports (host); global indices are shipped only when the rank holds a subset"}

    side = {}
    cpu = None
    if rank == 0 and cpu_state:
        cpu = cpu_baseline(prog, cpu_state["recs"], cpu_state["gidx"], lo, hi, args.cpu_records, batches[0][0])
        cpu_state.clear()
    nccl_ranks = ctx.stats()["nccl_ranks"]
    ctx.close()
    del src
    torch.cuda.empty_cache()
    if not args.no_side and args.workload == "config5" and args.scale == 1.0:
        for name in ("config3", "config4"):
            side[name] = side_workload(name, args, dev, stream, world, rank, hbm_gbs, peak_src, flags)
            torch.cuda.empty_cache()

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": "u8",
                "data": "synthetic (counter-based generator, generated on the device before each timed batch)",
                "config": {"workload": args.workload, "scale": args.scale, "buffer_overflow_ext": bool(args.bo),
                           "reporting": "dedup_first (ARB_F_DEDUP_FIRST)" if args.dedup else
                                        "raw (one report per faulting word-event, the oracle's canonical mode)",
                           "records_per_step": int(records_all), "word_events_per_step": int(word_events_all),
                           "access_word_events_per_step": int(access_all),
                           "access_word_events_per_s": access_all / (ms_per_step / 1e3),
                           "records_per_s": records_all / (ms_per_step / 1e3),
                           "range_word_events_per_step_rank0": int(s0["range_words"]),
                           "reports_per_step": int(reports_all), "reports_by_kind_rank0": s0["by_kind"][1:],
                           "time_batches": len(batches), "flushes_per_step_rank0": int(s0["flushes"]),
                           "rank_words": hi - lo, "batches_rank0": binfo,
                           "replay_steps_fast_sort_run_rank0": [int(s0["steps_fast"]), int(s0["steps_sort"]),
                                                                int(s0["steps_run"])],
                           "segments_rank0": int(s0["segments"]),
                           "chunks_all_fast_run_rank0": [int(s0["chunks"]), int(s0["chunks_fast"]), int(s0["chunks_run"])],
                           "run_merges_rank0": int(s0["run_merges"]),
                           "max_bucket_events_rank0": int(s0["max_bucket_events"]),
                           "replay_work_items_rank0": int(s0["work_items"]),
                           "hot_buckets_rank0": int(s0["hot_buckets"]),
                           "nccl": {"ranks": nccl_ranks, "exchanges_per_step_rank0": int(s0["exchanges"])},
                           "l2": "inputs larger than L2 (>= 1 GB of records per timed batch)",
                           "timing": "per batch: barrier + synchronize, CUDA events on the replay stream around "
                                     "the batch's flushes, max over ranks; step = sum over batches",
                           "bench_wall_s": round(t_wall, 1)},
                "clocks": clk, "e2e": e2e, "gpu_launches": int(launches_all),
                "roofline": roof, "cpu_baseline": cpu, "workloads": side or None}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
