#!/usr/bin/env python
"""Benchmark of the B200 ARBALEST replay (BASELINE.json metric: events/sec replayed
at 1/2/4/8 B200 and % of HBM roofline; vs CPU oracle).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload config5|config3|config4|config2]
    python -m torch.distributed.run --nproc-per-node N --master-addr 127.0.0.1 ... bench.py --gpus N
    python bench.py --impl reference ...     (the CPU oracle, timed on the host cores)

One step = one pass of the whole hot path (decode + partition, control
resolution, replay + classification, MIR join, report compaction, count
exchange) over the rank's batch of synthetic records, which are generated on the
device before timing.  Default workload: config 5 (address-sharded trace; weak
scaling: rank r replays shard r, ~1.1e9 records / ~1.25e9 word-events per rank).
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


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as fh:
            d = json.load(fh)
        return float(d["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


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
def make_program(name, scale):
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


def rank_batches(prog, rank, world, device, max_flush=1 << 29):
    """Generate the global trace on the device chunk by chunk, keep the records of
    this rank's shard (all control records + accesses touching its words), and
    cut the result into flushes at quiescent points.  Returns (recs, gidx, flushes,
    shard word range)."""
    import torch
    from gen import native
    from paper_conf_ipps_yuphs21_b200.shard import shard_range
    if prog.name == "config5" and world > 1:
        lo, hi = shard_range(prog.addr_base // 8, native.C5_SHARD_WORDS * native.C5_SHARDS, rank,
                             native.C5_SHARDS)
    elif prog.name == "config5":
        lo, hi = shard_range(prog.addr_base // 8, native.C5_SHARD_WORDS * native.C5_SHARDS, 0,
                             native.C5_SHARDS)
    else:
        lo, hi = shard_range(prog.addr_base // 8, prog.addr_bytes // 8, rank, world)
    # first pass: count per quiescent interval, second: generate into place
    q = prog.quiescent
    chunk = 1 << 27
    tmp = torch.empty((chunk, 2), dtype=torch.int64, device=device)
    kept_chunks, gidx_chunks, kept_upto = [], [], []
    total = 0
    start = 0
    while start < prog.n:
        cnt = min(chunk, prog.n - start)
        prog.fill_device(tmp, start, cnt)
        out = torch.empty((cnt, 2), dtype=torch.int64, device=device)
        gi = torch.empty(cnt, dtype=torch.int64, device=device)
        k = native.filter_device(tmp, cnt, lo, hi, start, out, gi)
        kept_chunks.append(out[:k].clone())
        gidx_chunks.append(gi[:k].clone())
        del out, gi
        total += k
        kept_upto.append((start + cnt, total))
        start += cnt
    del tmp
    recs = torch.cat(kept_chunks)
    gidx = torch.cat(gidx_chunks)
    del kept_chunks, gidx_chunks
    # flush cuts: local positions of quiescent global indices (searchsorted on gidx)
    qs = torch.tensor(q, dtype=torch.int64, device=device)
    local_q = torch.searchsorted(gidx, qs).cpu().numpy().tolist()
    cuts = [0]
    for a in local_q[1:]:
        if a - cuts[-1] > max_flush:
            # the previous quiescent point is the last legal cut before exceeding the limit
            prev = max(c for c in local_q if c <= cuts[-1] + max_flush)
            if prev > cuts[-1]:
                cuts.append(prev)
    if cuts[-1] != recs.shape[0]:
        cuts.append(recs.shape[0])
    flushes = [(a, b) for a, b in zip(cuts[:-1], cuts[1:]) if b > a]
    return recs, gidx, flushes, (lo, hi)


# ---------------------------------------------------------------------------
def run_reference(args):
    """--impl reference: the CPU oracle as it stands, on the host cores, on a bounded
    sample of the same workload (rank 0 only)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    from gen import native
    prog = make_program(args.workload, args.scale)
    lo = prog.addr_base // 8
    hi = lo + (native.C5_SHARD_WORDS if prog.name == "config5" else prog.addr_bytes // 8)
    sample = args.ref_sample
    rec, gi = prog.filter_host(word_lo=lo, word_hi=hi, start=0, count=min(prog.n, sample * 8))
    cut = quiescent_prefix(prog, gi, sample)
    rec, gi = rec[:cut], gi[:cut]
    times, evs = [], 0
    for s in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        r = oracle.replay(rec, lo * 8, (hi - lo) * 8, global_index=gi, want_shadow=False)
        dt = time.perf_counter() - t0
        assert r.rc == 0
        if s >= args.warmup:
            times.append(dt)
            evs = r.stats["word_events"]
    v = evs / float(np.mean(times))
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * float(np.mean(times)),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u8",
            "data": "synthetic",
            "config": {"workload": args.workload, "sample_records": int(rec.shape[0]),
                       "sample_word_events": int(evs)},
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": 1, "kind": "oracle",
                             "sample": f"first {rec.shape[0]} records of shard 0 of {args.workload}"},
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


def cpu_baseline(prog, recs_dev, gidx_dev, lo, hi, budget_records):
    import oracle
    n = quiescent_prefix(prog, gidx_dev.cpu().numpy(), min(budget_records, recs_dev.shape[0]))
    rec = recs_dev[:n].cpu().numpy().view(np.uint64)
    gi = gidx_dev[:n].cpu().numpy().view(np.uint64)
    t0 = time.perf_counter()
    r = oracle.replay(rec, lo * 8, (hi - lo) * 8, global_index=gi, want_shadow=False)
    dt = time.perf_counter() - t0
    assert r.rc == 0, r.rc
    return {"value": r.stats["word_events"] / dt, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"first {n} records of rank 0's batch ({r.stats['word_events']} word-events, "
                      f"{dt:.1f} s, single-threaded plain C)"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="config5")
    ap.add_argument("--scale", type=float, default=1.0)
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--bo", action="store_true", help="enable the buffer-overflow extension (ARB_F_BO, Z20)")
    ap.add_argument("--cpu-records", type=int, default=300_000_000)
    ap.add_argument("--ref-sample", type=int, default=15_000_000)
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist
    from paper_conf_ipps_yuphs21_b200 import Context, ARB_F_TIMING, ARB_F_BO, reports_to_triples
    from paper_conf_ipps_yuphs21_b200.shard import nccl_unique_id

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    hbm_gbs, peak_src = peaks()

    prog = make_program(args.workload, args.scale)
    t_gen = time.perf_counter()
    recs, gidx, flushes, (lo, hi) = rank_batches(prog, rank, world, dev)
    if world > 1:
        # every arb_flush exchanges the report counts (ncclAllGather), so all ranks
        # must flush equally often: pad the shorter schedules with empty flushes
        nf = torch.tensor([len(flushes)], dtype=torch.int64, device=dev)
        dist.all_reduce(nf, op=dist.ReduceOp.MAX)
        flushes = flushes + [(recs.shape[0], recs.shape[0])] * (int(nf.item()) - len(flushes))
    torch.cuda.synchronize()
    t_gen = time.perf_counter() - t_gen

    uid = None
    if world > 1:
        buf = torch.zeros(128, dtype=torch.uint8, device=dev)
        if rank == 0:
            buf.copy_(torch.frombuffer(bytearray(nccl_unique_id()), dtype=torch.uint8))
        dist.broadcast(buf, 0)
        uid = bytes(buf.cpu().numpy().tobytes())
    ctx = Context(lo * 8, (hi - lo) * 8, device=local, rank=rank, world=world, nccl_unique_id=uid,
                  flags=ARB_F_TIMING | (ARB_F_BO if args.bo else 0), report_capacity=1 << 25)
    stream = torch.cuda.Stream(device=dev)

    def one_step(collect=False):
        st_acc = {"access_words": 0, "range_words": 0, "reports": 0, "launches": 0, "ms_partition": 0.0,
                  "ms_replay": 0.0, "ms_mir": 0.0, "ms_reports": 0.0, "ms_control": 0.0, "ms_total": 0.0,
                  "ms_sample": 0.0, "ms_segsort": 0.0, "ms_host_control": 0.0, "records": 0,
                  "steps_fast": 0, "steps_sort": 0, "max_bucket_events": 0, "work_items": 0,
                  "hot_buckets": 0,
                  "by_kind": [0, 0, 0, 0]}
        for (a, b) in flushes:
            ctx.submit_events(recs[a:b], global_index=gidx[a:b], stream=stream)
            rc, n, off = ctx.flush(stream=stream)
            st = ctx.stats()
            for k in ("access_words", "range_words", "reports", "records", "ms_partition", "ms_replay",
                      "ms_mir", "ms_reports", "ms_control", "ms_total", "ms_sample", "ms_segsort",
                      "ms_host_control", "steps_fast", "steps_sort", "work_items",
                      "hot_buckets"):
                st_acc[k] += st[k]
            st_acc["max_bucket_events"] = max(st_acc["max_bucket_events"], st["max_bucket_events"])
            st_acc["launches"] += st["kernel_launches"]
            for k in range(4):
                st_acc["by_kind"][k] += st["reports_by_kind"][k]
        return st_acc

    # ---- warm-up ------------------------------------------------------------
    for _ in range(args.warmup):
        first = one_step()
    torch.cuda.synchronize()
    # ---- timed region -----------------------------------------------------------
    clocks = ClockSampler(local)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks.start()
    time.sleep(0.3)
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    ev0.record(stream)
    per_step = []
    for _ in range(args.steps):
        per_step.append(one_step())
    ev1.record(stream)
    torch.cuda.synchronize()
    clk = clocks.stop()
    if world > 1:
        dist.barrier()
    ms = ev0.elapsed_time(ev1)
    t = torch.tensor([ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_max = float(t.item())
    s0 = per_step[-1]
    word_events_rank = s0["access_words"] + s0["range_words"]
    tot = torch.tensor([word_events_rank, s0["records"], s0["reports"]], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(tot)
    word_events_all, records_all, reports_all = [float(x) for x in tot.tolist()]
    value = word_events_all * args.steps / (ms_max / 1e3)
    ms_per_step = ms_max / args.steps

    n_busy = max(1, sum(1 for a, b in flushes if b > a))   # non-empty flushes (kernel launches)
    # ---- roofline: B_alg = 16 R + 2 W + 16 Rep -------------------------
    W = sum(prog.distinct_words(lo, hi, [(int(gidx[a].item()), int(gidx[b - 1].item()) + 1)
                                         for a, b in flushes if b > a]))
    b_alg = 16 * s0["records"] + 2 * W + 16 * s0["reports"]
    step_ms_lib = s0["ms_total"]
    phases = {"k_sample+balance": s0["ms_sample"], "k_partition": s0["ms_partition"] - s0["ms_sample"],
              "k_replay": s0["ms_replay"], "k_mir": s0["ms_mir"],
              "report_compaction": s0["ms_reports"], "control_plane": s0["ms_control"],
              "segment_sort (in control_plane)": s0["ms_segsort"],
              "host_control_wall (in control_plane)": s0["ms_host_control"]}
    dom = max(("k_partition", "k_replay"), key=lambda k: phases[k])
    # algorithmic bytes of each kernel: the partition kernel reads every
    # record once (16 R); the replay owns the shadow term (2 W) and the report writes (16 Rep)
    alg = {"k_partition": 16 * s0["records"], "k_replay": 2 * W + 16 * s0["reports"]}
    achieved = alg[dom] / (phases[dom] / 1e3) / 1e9 if phases[dom] > 0 else 0.0
    # DRAM traffic of the dominant kernel from the committed `ncu --set full`
    # capture (profiles/traffic.json), scaled per launch to this step's records
    traffic = None
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as fh:
            tj = json.load(fh)[dom]
        traffic = tj["dram_bytes_per_launch"] / tj["records_in_launch"] * s0["records"] / n_busy
    except Exception:
        pass
    kern = {}
    for k in ("k_partition", "k_replay"):
        ach = alg[k] / (phases[k] / 1e3) / 1e9 if phases[k] > 0 else 0.0
        kern[k] = {"ms_per_step": phases[k], "alg_bytes_per_step": alg[k], "achieved": ach, "frac": ach / hbm_gbs}
        try:
            with open(os.path.join(ROOT, "profiles", "traffic.json")) as fh:
                tk = json.load(fh)[k]
            kern[k]["ncu_dram_bytes_per_record"] = tk["dram_bytes_per_launch"] / tk["records_in_launch"]
        except Exception:
            pass
    roof = {"bound": "hbm", "kernel": dom, "achieved": achieved, "peak": hbm_gbs, "unit": "GB/s",
            "frac": achieved / hbm_gbs, "traffic": traffic, "traffic_unit": "bytes per launch (ncu)",
            "alg_bytes_per_launch": alg[dom] / n_busy, "peak_source": peak_src,
            "kernel_ms_per_step": phases[dom], "phase_ms_per_step": phases, "kernels": kern,
            "path": {"b_alg_bytes_per_step": b_alg, "achieved": b_alg / (ms_per_step / 1e3) / 1e9,
                     "frac": b_alg / (ms_per_step / 1e3) / 1e9 / hbm_gbs}}
    if dom == "k_replay":
        roof["note"] = ("k_replay is instruction-issue bound (ncu: ~68 % issue active, ~27 % of DRAM peak, "
                        "profiles/); its algorithmic bytes are the shadow (2 B per distinct word) and the "
                        "reports (16 B each), SURVEY §8(d) -- the 8-B partition events it reads are design "
                        "overhead -- so its HBM fraction is small by construction; kernels.k_partition "
                        "(reads the trace, 16 B/record) and path (B_alg / step time) carry the HBM roofline")

    # ---- e2e: host buffers through the public API ----------------------------------
    e2e = None
    if not args.no_e2e:
        h_rec = torch.empty(recs.shape, dtype=recs.dtype, pin_memory=True)
        h_gi = torch.empty(gidx.shape, dtype=gidx.dtype, pin_memory=True)
        h_rec.copy_(recs)
        h_gi.copy_(gidx)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        d2h = 0
        for _ in range(args.e2e_steps):
            for (a, b) in flushes:
                ctx.submit_events(h_rec[a:b], global_index=h_gi[a:b], stream=stream)
                rc, n, off = ctx.flush(stream=stream)
                rep = ctx.get_reports(n)
                d2h += rep.nbytes + 16
        torch.cuda.synchronize()
        dt = torch.tensor([time.perf_counter() - t0], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(dt, op=dist.ReduceOp.MAX)
        e2e = {"value": word_events_all * args.e2e_steps / float(dt.item()), "unit": UNIT,
               "h2d_bytes_per_step": int(recs.numel() * 8 + gidx.numel() * 8),
               "d2h_bytes_per_step": int(d2h // args.e2e_steps)}
        del h_rec, h_gi

    if rank == 0:
        cpu = None
        if not args.no_cpu and world == 1:        # the oracle baseline is an N = 1 figure
            cpu = cpu_baseline(prog, recs, gidx, lo, hi, args.cpu_records)
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": "u8", "data": "synthetic",
                "config": {"workload": args.workload, "scale": args.scale, "buffer_overflow_ext": bool(args.bo),
                           "records_per_step": int(records_all), "word_events_per_step": int(word_events_all),
                           "access_word_events_per_step_rank0": int(s0["access_words"]),
                           "range_word_events_per_step_rank0": int(s0["range_words"]),
                           "reports_per_step": int(reports_all), "reports_by_kind_rank0": s0["by_kind"][1:],
                           "flushes_per_step_rank0": n_busy, "shard_words": hi - lo,
                           "replay_steps_fast_sort_rank0": [int(s0["steps_fast"]), int(s0["steps_sort"])],
                           "max_bucket_events_rank0": int(s0["max_bucket_events"]),
                           "replay_work_items_rank0": int(s0["work_items"]),
                           "hot_buckets_rank0": int(s0["hot_buckets"]),
                           "l2": "inputs larger than L2 (>= 16 GB of records per step)",
                           "generation_s": round(t_gen, 2)},
                "clocks": clk, "e2e": e2e, "gpu_launches": int(sum(s["launches"] for s in per_step)),
                "roofline": roof, "cpu_baseline": cpu}
        print(json.dumps(line), flush=True)
    ctx.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
