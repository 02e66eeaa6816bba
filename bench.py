#!/usr/bin/env python
"""Benchmark of the LC-style codec hot path on B200.

A step = compress + decompress, through the C ABI with device-resident data,
of every codec on its field of the workload (BASELINE.json configs[1] for the
SP codecs — CESM-ATM-shaped 1800×3600 f32 fields T and U — and configs[2]'s
Miranda-shaped 256×384×384 f64 density field for the DP codecs, so all §8(a)
rows run every step). The L2 is flushed (256 MiB write) before every timed
call; each call is timed with CUDA events on the launching stream.

Metric: uncompressed GB/s (10^9 B/s) = Σ uncompressed bytes moved through
compress and decompress ÷ Σ device time, plus per-codec compress/decompress
GB/s, ratio and HBM-roofline fraction. Multi-GPU (torchrun): weak scaling,
each rank owns a contiguous chunk range of one global stream per field (the
fields are generated as sub-blocks of N× larger global fields), compresses it
with lcf_compress_shard and all-gathers the per-rank payload byte counts over
NCCL (the only exchange).

`--impl reference` times the CPU oracle (oracle/) on a bounded sample of the
same workload — the only reference this paper-only tier has.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

# (config, fields, codecs): BASELINE.json configs[1] (CESM-ATM-shaped) and
# configs[3] (NYX-shaped 512³ and the HACC-like 1-D arrays — the largest
# single-GPU SP configuration) for the SP codecs; configs[2] (Miranda-shaped)
# for the DP codecs, with `rt_density` the field whose exact repeats FCM finds
FIELD_SETS = (
    ("cesm_1800x3600_f32", ("T", "U"), ("SPspeed", "SPratio")),
    ("nyx_512x512x512_f32", ("baryon_density", "velocity"), ("SPspeed", "SPratio")),
    ("hacc_280953867_f32", ("xx", "vx"), ("SPspeed", "SPratio")),
    ("miranda_256x384x384_f64", ("density", "rt_density"), ("DPspeed", "DPratio")),
)
WORKLOAD = " + ".join(f"{cfg}[{','.join(names)}]:{','.join(codecs)}" for cfg, names, codecs in FIELD_SETS)
ALL_CODECS = ("SPspeed", "SPratio", "DPspeed", "DPratio")
L2_FLUSH_BYTES = 256 << 20


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


class ClockSampler:
    """SM clock and throttle reasons polled through NVML every ~2 ms while the
    timed region runs (the same counters `nvidia-smi --query-gpu=clocks.sm,
    clocks_event_reasons.*` reads)."""
    REASONS = {0x8: "hw_slowdown", 0x40: "sw_thermal_slowdown", 0x20: "hw_thermal_slowdown",
               0x4: "sw_power_cap", 0x80: "hw_power_brake_slowdown"}

    def __init__(self, index: int):
        self.index, self.sm, self.bits, self.max_mhz, self.stop = index, [], 0, None, False

    def __enter__(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.t = threading.Thread(target=self._poll, daemon=True)
            self.t.start()
        except Exception as e:  # noqa: BLE001
            self.nv = None
            self.err = repr(e)
        return self

    def _poll(self):
        nv = self.nv
        while not self.stop:
            try:
                self.sm.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                self.bits |= nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
            except Exception:  # noqa: BLE001
                pass
            time.sleep(0.002)

    def __exit__(self, *exc):
        self.stop = True
        if self.nv:
            self.t.join(timeout=1)

    def summary(self):
        if not self.nv or not self.sm:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": ["unavailable"]}
        reasons = sorted(v for k, v in self.REASONS.items() if self.bits & k)
        return {"sm_mhz": statistics.median(self.sm), "sm_max_mhz": self.max_mhz, "reasons": reasons,
                "samples": len(self.sm)}


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def replica_bytes(cfg):
    from paper_conf_asplos_azamifb25_b200 import datagen
    _, shape, dtype, _ = datagen.CONFIGS[cfg]
    n = 1
    for d in shape:
        n *= d
    return n * (4 if dtype == torch.float32 else 8)


def make_fields(world, rank, device, sets=None):
    """Per-field inputs. N = 1: the config's field. N > 1 (weak scaling): the
    global input is the concatenation of N independent replicas of the field;
    chunk-local codecs get this rank's chunk-range shard of it (generated from
    the ≤ 3 replicas the shard overlaps), DPratio (whole-array FCM) gets
    replica `rank` whole."""
    from paper_conf_asplos_azamifb25_b200 import datagen, sharded
    fields = []
    for cfg, names, codecs in (sets or FIELD_SETS):
        rb = replica_bytes(cfg)
        for nm in names:
            own = datagen.field(cfg, nm, device=device, replica=rank).reshape(-1)
            wdt = torch.int32 if own.dtype == torch.float32 else torch.int64
            own = own.view(wdt)
            shard, total = own, rb
            if world > 1:
                total = world * rb
                off, ln = sharded.shard_bytes(total, world, rank)
                r0, r1 = off // rb, (off + max(ln, 1) - 1) // rb
                parts = [own if r == rank else datagen.field(cfg, nm, device=device, replica=r).reshape(-1).view(wdt)
                         for r in range(r0, r1 + 1)]
                whole = torch.cat(parts) if len(parts) > 1 else parts[0]
                shard = whole.view(torch.uint8)[off - r0 * rb:off - r0 * rb + ln].view(wdt).clone()
                del parts, whole
            for codec in codecs:
                x = own if (codec == "DPratio" or world == 1) else shard
                fields.append((cfg, nm, codec, x, total))
            torch.cuda.empty_cache()
    return fields


def kernel_traffic():
    """dram__bytes_read + dram__bytes_write per launch of each kernel on this
    workload, from the newest committed `ncu --set full` summary
    (profiles/<round>_kernel_traffic.json, scripts/profile_round.sh)."""
    import glob
    files = sorted(glob.glob(os.path.join(ROOT, "profiles", "*_kernel_traffic.json")))
    if not files:
        return {}
    with open(files[-1]) as f:
        d = json.load(f)
    return {k.split(":", 1)[1]: v["dram_bytes_per_launch"] for k, v in d.items()}


def kernel_bytes(j):
    """Algorithmic bytes of every kernel a job's compress and decompress
    launch, summed over the job's launches of that kernel (DESIGN.md §6 gives
    the per-launch figures): the I/O the method itself must move."""
    n, sb, codec = j["nbytes"], j["sbytes"], j["codec"]
    words = n // (4 if codec.startswith("SP") else 8)
    io = n + sb
    if codec == "SPspeed":
        return {"speed_encode_u32": io, "speed_decode_u32": io}
    if codec == "DPspeed":
        return {"speed_encode_u64": io, "speed_decode_u64": io}
    if codec == "SPratio":
        return {"spratio_encode": io, "spratio_decode": io}
    tiles = -(-words // 16384)
    # the sort kernels launch once per radix pass (two passes per job)
    return {"fcm_sort_ghist": 8 * words,              # x in (both passes' digit totals in one read)
            "fcm_sort_hist": 2 * 8 * words,           # (LCF_ONESWEEP=0 build) x or pass-1 records in
            "fcm_sort_scan": 2 * 8 * 1024 * tiles,    # (LCF_ONESWEEP=0 build) the tile × digit count matrix
            "fcm_sort_scatter": 2 * 16 * words,       # 8-byte records (or x) in, records out, per pass
            "fcm_match": 8 * words,                   # sorted records in (candidates scattered)
            "fcm_verify": 4 * words,                  # the candidate array in (x read only at candidates)
            "dp_walk_nodes": 0,                       # (data-dependent: the chain-node list)
            "dp_gather_nodes": 0,
            "dpratio_encode": 12 * words + sb,        # x + distances in, stream out
            "dpratio_decode": sb + n,                 # stream in, x out
            "dp_find_roots": words // 8,              # the pending bitmap (the walks are data-dependent)
            "dp_gather_leaves": words // 8,
            "dp_gather_roots": words // 8}


def compress_op(lcf, j):
    """Compress this rank's input; in sharded mode also all-gather the local
    payload byte count (a device u64 at header byte 24) — the single
    exchange of SURVEY §8(e), stream-ordered, no host sync."""
    lcf.lcf_compress(j["codec"], None, j["x"], j["nbytes"], j["s"], j["cap"], sync=False)
    if j["counts"] is not None:
        torch.distributed.all_gather_into_tensor(j["counts"], j["s"][24:32].view(torch.int64))


class Timer:
    def __init__(self):
        self.flush = torch.empty(L2_FLUSH_BYTES, dtype=torch.uint8, device="cuda")

    def time(self, fn):
        self.flush.fill_(1)  # evict the L2 (126 MB) before every timed call
        st = torch.cuda.current_stream()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(st)
        fn()
        b.record(st)
        return a, b


def run_lcf(args):
    from paper_conf_asplos_azamifb25_b200 import lcf
    world, rank, local = dist_env()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=dev)
    codecs = [c for c in args.codecs.split(",") if c]
    fields = make_fields(world, rank, dev)
    stream = torch.cuda.current_stream()

    # one job per (codec, field): buffers allocated once, outside the timed region
    jobs = []
    for cfg, nm, codec, x, total in fields:
        if codec not in codecs:
            continue
        nbytes = x.numel() * x.element_size()
        cap = lcf.lcf_max_compressed_size(codec, None, nbytes)
        s = torch.empty(cap, dtype=torch.uint8, device=dev)
        y = torch.empty_like(x)
        n = lcf.lcf_compress(codec, None, x, nbytes, s, cap)  # every codec must run: no skip
        lcf.lcf_decompress(codec, None, s, n, y, nbytes)
        assert torch.equal(x, y), f"{codec}/{nm}: round trip failed"
        sharded_job = world > 1 and codec != "DPratio"
        counts = torch.empty(world, dtype=torch.int64, device=dev) if sharded_job else None
        jobs.append({"codec": codec, "field": f"{cfg}/{nm}", "x": x, "s": s, "y": y, "cap": cap,
                     "nbytes": nbytes, "sbytes": n, "ct": [], "dt": [], "counts": counts})
    timer = Timer()

    def step(record):
        evs = []
        for j in jobs:
            c = timer.time(lambda j=j: compress_op(lcf, j))
            d = timer.time(lambda j=j: lcf.lcf_decompress(j["codec"], None, j["s"], j["sbytes"], j["y"],
                                                          j["nbytes"], sync=False))
            evs.append((j, c, d))
        if record:
            torch.cuda.synchronize()
            for j, c, d in evs:
                j["ct"].append(c[0].elapsed_time(c[1]))
                j["dt"].append(d[0].elapsed_time(d[1]))

    for _ in range(args.warmup):
        step(False)
    lcf.lcf_check_stream()
    torch.cuda.synchronize()
    if world > 1:
        torch.distributed.barrier()
    launches0 = lcf.lcf_launch_count()
    with ClockSampler(local) as clk:
        t0 = time.perf_counter()
        for _ in range(args.steps):
            step(True)
        torch.cuda.synchronize()
        wall = time.perf_counter() - t0
    launches = lcf.lcf_launch_count() - launches0
    lcf.lcf_check_stream()
    # per-kernel live timing in a separate pass of the same steps (CUDA events
    # around every library launch would perturb the timed region above)
    lcf.lcf_profile_report()  # clear
    lcf.lcf_profile_enable(True)
    for _ in range(args.steps):
        step(False)
    torch.cuda.synchronize()
    lcf.lcf_profile_enable(False)
    ktimes = lcf.lcf_profile_report()
    lcf.lcf_check_stream()
    for j in jobs:  # the timed outputs are still exact
        assert torch.equal(j["x"], j["y"]), j["codec"]

    hbm, peak_kind = peaks()
    per_codec, tot_bytes, tot_ms = {}, 0, 0.0
    kbytes = {}
    for j in jobs:
        ct, dt = statistics.median(j["ct"]), statistics.median(j["dt"])
        moved = j["nbytes"] + j["sbytes"]
        key = f"{j['codec']}:{j['field']}"
        per_codec[key] = {
            "compress_gbs": j["nbytes"] / ct / 1e6, "decompress_gbs": j["nbytes"] / dt / 1e6,
            "ratio": j["nbytes"] / j["sbytes"], "compress_ms": ct, "decompress_ms": dt,
            "compress_roofline_frac": moved / ct / 1e6 / hbm, "decompress_roofline_frac": moved / dt / 1e6 / hbm,
        }
        tot_bytes += 2 * j["nbytes"]
        tot_ms += ct + dt
        for name, b in kernel_bytes(j).items():
            kbytes[name] = kbytes.get(name, 0) + b * args.steps
    # per-kernel live timing (CUDA events around every library launch, timed region only)
    kernels = {}
    for name, (cnt, ms) in ktimes.items():
        if name not in kbytes or ms <= 0:
            continue
        if kbytes[name] == 0:  # data-dependent kernels: time share only
            kernels[name] = {"launches": cnt, "avg_ms": ms / cnt, "share": 0.0, "achieved_gbs": None, "frac": None}
            continue
        kernels[name] = {"launches": cnt, "avg_ms": ms / cnt, "share": 0.0,
                         "achieved_gbs": kbytes[name] / ms / 1e6, "frac": kbytes[name] / ms / 1e6 / hbm}
    ksum = sum(ms for _, ms in ktimes.values()) or 1.0
    for name in kernels:
        kernels[name]["share"] = ktimes[name][1] / ksum
    own = {k: v for k, v in kernels.items() if not k.startswith("cub_") and v["frac"] is not None}
    dom = max(own, key=lambda k: ktimes[k][1]) if own else None
    roofline = None
    traffic = kernel_traffic()
    if dom:
        d = kernels[dom]
        roofline = {"bound": "hbm", "achieved": d["achieved_gbs"], "peak": hbm, "unit": "GB/s", "frac": d["frac"],
                    "traffic": traffic.get(dom), "kernel": dom, "peak_kind": peak_kind,
                    "algorithmic_bytes_per_launch": kbytes[dom] / max(1, d["launches"]),
                    "avg_launch_ms": d["avg_ms"], "share_of_step": d["share"],
                    "timing": "CUDA events around each launch on its stream, in a second pass of the same steps"}
    value = tot_bytes / tot_ms / 1e6
    # aggregate over ranks: weak scaling, max step time
    ms_step = tot_ms
    if world > 1:
        tt = torch.tensor([ms_step], device=dev)
        torch.distributed.all_reduce(tt, op=torch.distributed.ReduceOp.MAX)
        ms_step = float(tt.item())
        value = world * tot_bytes / ms_step / 1e6

    transfer = None
    if world > 1 and args.transfer:  # (on by default at N ≥ 2)
        try:
            transfer = run_transfer(jobs, rank, dev)
        except Exception as e:  # a measurement extra: never fail the bench line for it
            print(f"[bench] transfer measurement failed: {e!r}", file=sys.stderr)
    e2e = run_e2e(lcf, jobs, args, world)
    cpu = run_cpu_baseline(jobs) if (rank == 0 and world == 1 and not args.no_cpu_baseline) else None
    cpu_codec = run_cpu_codec(jobs) if (rank == 0 and world == 1 and not args.no_cpu_baseline) else None
    if rank == 0:
        line = {
            "metric": "compress+decompress throughput (uncompressed GB/s)", "value": value, "unit": "GB/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_step,
            "wall_ms_per_step": wall / args.steps * 1e3, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u32/u64 (f32/f64 bits)", "data": "synthetic",
            "config": {"workload": WORKLOAD, "l2": "flushed (256 MiB write) before every timed call",
                       "parallelism": f"chunk-range shards x{world}" if world > 1 else "single GPU"},
            "per_codec": per_codec, "kernels": kernels, "roofline": roofline, "cpu_baseline": cpu, "cpu_codec": cpu_codec, "e2e": e2e,
            "gpu_launches": launches, "clocks": clk.summary(),
        }
        if transfer is not None:
            line["transfer"] = transfer
        print(json.dumps(line))
    if world > 1:
        torch.distributed.destroy_process_group()


def run_transfer(jobs, rank, dev, reps: int = 3):
    """NEXT-3 (transfer.py): rank 0 → rank 1, the raw words (dist.send), the
    compressed sub-streams (send_compressed / recv_compressed, NCCL payload
    messages) and the fused form (transfer.P2PChannel: the compress kernels
    write the stream into rank 1's buffer over NVLink, rank 1 decompresses),
    per job. GB/s = uncompressed bytes / time, timed on the device (events on
    each rank's current stream), max over the pair, median of `reps`."""
    import statistics
    import torch.distributed as dist
    from paper_conf_asplos_azamifb25_b200 import transfer as tr
    out = []
    for j in jobs:
        x = j["x"]
        # the receiver sizes its buffer from the sender's (shards of one stream differ in length)
        nel = torch.tensor([x.numel()], dtype=torch.int64, device=dev)
        if rank == 0:
            dist.send(nel, 1)
        elif rank == 1:
            dist.recv(nel, 0)
        buf = torch.empty(int(nel.item()), dtype=x.dtype, device=dev)
        ch = tr.P2PChannel(0, 1, j["codec"], int(nel.item()) * x.element_size()) if rank < 2 else None
        res = {}
        for mode in ("raw", "compressed", "fused_p2p"):
            if mode == "compressed" and j["codec"] == "DPratio":
                continue
            ts = []
            for _ in range(reps):
                dist.barrier()
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                if rank == 0:
                    if mode == "raw":
                        dist.send(x, 1)
                    elif mode == "compressed":
                        tr.send_compressed(x, 1, j["codec"])
                    else:
                        ch.send(x)
                elif rank == 1:
                    if mode == "raw":
                        dist.recv(buf, 0)
                    elif mode == "compressed":
                        tr.recv_compressed(0, j["codec"], device=dev)
                    else:
                        ch.recv(buf)
                e1.record()
                torch.cuda.synchronize()
                t = torch.tensor([e0.elapsed_time(e1) if rank < 2 else 0.0], device=dev)
                dist.all_reduce(t, op=dist.ReduceOp.MAX)
                ts.append(float(t.item()))
            res[mode] = j["nbytes"] / statistics.median(ts) / 1e6
        if ch is not None:
            ch.close()
        dist.barrier()
        out.append({"codec": j["codec"], "field": j["field"], "bytes": j["nbytes"], "raw_gbs": res["raw"],
                    "compressed_gbs": res.get("compressed"), "fused_p2p_gbs": res["fused_p2p"],
                    "ratio": j["nbytes"] / j["sbytes"]})
    return {"pair": "rank 0 -> rank 1", "timing": "device events, max over the pair, median of 3",
            "modes": {"raw": "NCCL send/recv of the words",
                      "compressed": "slice-pipelined compressed sub-streams over NCCL send/recv",
                      "fused_p2p": "compress kernels store into rank 1's buffer over NVLink (CUDA IPC), "
                                   "then rank 1 decompresses"},
            "jobs": out}


def run_e2e(lcf, jobs, args, world=1):
    """Same metric through lcf_compress_host / lcf_decompress_host (pinned
    host buffers; H2D of the step's inputs and D2H of its results inside),
    on every rank at once; the step time is the max over ranks.

    The jobs run as a two-stage pipeline, the way a user streams fields
    through the host API: one host thread compresses job after job on its own
    CUDA stream while a second thread decompresses each finished stream on
    another (per-stream workspaces make the calls independent, include/lcf.h).
    Compression is bound by its H2D copy of the raw field and decompression by
    its D2H copy of the restored field, so the two stages use both directions
    of the full-duplex PCIe link. Jobs go largest first (the last, smallest
    decompression is the pipeline's tail). Every stream and restored field is
    checked in an untimed pass after the timed steps."""
    import queue
    import threading
    order = sorted(range(len(jobs)), key=lambda i: -jobs[i]["nbytes"])
    xin, yout, host = {}, {}, []
    for i in order:
        j = jobs[i]
        key = j["x"].data_ptr()
        if key not in xin:  # input and restored field: one pinned pair per field
            hx = torch.empty(j["nbytes"], dtype=torch.uint8, pin_memory=True)
            hx.copy_(j["x"].view(torch.uint8).cpu())
            xin[key] = hx
            yout[key] = torch.empty(j["nbytes"], dtype=torch.uint8, pin_memory=True)
        # each job its own stream buffer: the compressor runs ahead of the decompressor
        host.append((j, xin[key], torch.empty(j["cap"], dtype=torch.uint8, pin_memory=True), yout[key]))
    sc, sd = torch.cuda.Stream(), torch.cuda.Stream()

    def step(check=False):
        q, err, sizes = queue.Queue(), [], {}

        def compressor():
            try:
                for idx, (j, hx, hs, _) in enumerate(host):
                    q.put((idx, lcf.lcf_compress_host(j["codec"], None, hx, j["nbytes"], hs, hs.numel(), stream=sc)))
            except BaseException as e:  # re-raised by the caller
                err.append(e)
            q.put(None)

        th = threading.Thread(target=compressor)
        th.start()
        while True:
            item = q.get()
            if item is None:
                break
            idx, n = item
            j, hx, hs, hy = host[idx]
            m = lcf.lcf_decompress_host(j["codec"], None, hs, n, hy, j["nbytes"], stream=sd)
            sizes[idx] = (n, m)
            if check:
                assert m == j["nbytes"] and torch.equal(hx, hy), j["codec"]
        th.join()
        if err:
            raise err[0]
        return sizes

    times = []
    iters = 1 + min(3, max(1, args.steps))  # one warm-up, ≤ 3 timed (PCIe-bound, seconds each)
    for it in range(iters):
        torch.cuda.synchronize()
        if world > 1:
            torch.distributed.barrier()
        t0 = time.perf_counter()
        sizes = step()
        times.append(time.perf_counter() - t0)
    step(check=True)
    h2d = sum(j["nbytes"] + sizes[i][0] for i, (j, *_) in enumerate(host))
    d2h = sum(sizes[i][0] + sizes[i][1] for i in range(len(host)))
    t = statistics.median(times[1:])
    if world > 1:
        tt = torch.tensor([t], device="cuda")
        torch.distributed.all_reduce(tt, op=torch.distributed.ReduceOp.MAX)
        t = float(tt.item())
    total = world * sum(2 * j["nbytes"] for j, *_ in host)
    return {"value": total / t / 1e9, "unit": "GB/s", "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
            "ms_per_step": t * 1e3, "api": "lcf_compress_host + lcf_decompress_host",
            "timing": "host wall clock per step, median of 3 after 1 warm-up; compression of job j+1 and "
                      "decompression of job j overlap (two host threads, one CUDA stream each: full-duplex PCIe)"
                      + (", max over ranks; bytes per step are rank 0's" if world > 1 else "")}


def _host_words(j, nbytes):
    words = j["x"][: nbytes // j["x"].element_size()].cpu().numpy()
    return words.view(np.uint32 if words.dtype == np.int32 else np.uint64)


def run_cpu_baseline(jobs, budget_s: float = 12.0):
    """The oracle as it stands on a bounded sample of the workload: the first
    4 MiB of every (codec, field) job, single-threaded, repeated up to the
    budget; plus the same oracle functions run chunk-parallel over all host
    cores on the first 64 MiB of every chunk-local job — each
    thread compresses and decompresses its own chunk range as an independent
    stream (chunks are context-free, L104); DPratio's FCM is a whole-array
    pass, so it has no chunk-parallel oracle figure."""
    import oracle
    from concurrent.futures import ThreadPoolExecutor
    oracle.lib()
    sample_bytes = 4 << 20
    samples = [(j["codec"], _host_words(j, sample_bytes)) for j in jobs]
    done_bytes, spent, reps = 0, 0.0, 0
    while reps < 4 and (reps == 0 or spent * (reps + 1) / reps <= budget_s):
        for codec, words in samples:
            t0 = time.perf_counter()
            s = oracle.compress(codec, words)
            y = oracle.decompress(codec, s)
            spent += time.perf_counter() - t0
            done_bytes += 2 * words.nbytes
            if reps == 0:
                assert np.array_equal(y, words)
        reps += 1
    out = {"value": done_bytes / spent / 1e9, "unit": "GB/s", "cores": 1, "kind": "oracle",
           "sample": f"first {sample_bytes >> 20} MiB of every (codec, field) of the workload, compress+decompress, "
                     f"x{reps}; {spent:.1f} s single-threaded"}
    nt = os.cpu_count() or 1
    big = [(j["codec"], _host_words(j, 64 << 20)) for j in jobs if j["codec"] != "DPratio"]
    work = []
    for codec, words in big:
        cw = 16384 // words.itemsize
        nc = -(-len(words) // cw)
        per = -(-nc // nt)
        work += [(codec, words[c * cw:(c + per) * cw]) for c in range(0, nc, per)]

    def one(item):
        codec, w = item
        return np.array_equal(oracle.decompress(codec, oracle.compress(codec, w)), w)

    t0 = time.perf_counter()
    with ThreadPoolExecutor(max_workers=nt) as ex:
        ok = all(ex.map(one, work))
    t = time.perf_counter() - t0
    assert ok
    moved = 2 * sum(w.nbytes for _, w in big)
    out["multicore"] = {"value": moved / t / 1e9, "unit": "GB/s", "cores": nt, "kind": "oracle, chunk-parallel",
                        "sample": "first 64 MiB of every SPspeed/SPratio/DPspeed job, compress+decompress, "
                                  f"{nt} threads over chunk ranges; {t:.1f} s"}
    return out


CPU_CODEC_FIELDS = ("cesm_1800x3600_f32/T", "cesm_1800x3600_f32/U", "miranda_256x384x384_f64/density",
                    "miranda_256x384x384_f64/rt_density")


def run_cpu_codec(jobs):
    """The multi-threaded CPU codec (liblcf_cpu.so) on the
    CESM and Miranda jobs of the workload (whole fields; the NYX/HACC jobs are
    left out to bound the run), one step, all host cores: same metric; its
    streams must be the GPU's bytes (the paper's CPU/GPU compatibility, L354)."""
    jobs = [j for j in jobs if j["field"] in CPU_CODEC_FIELDS]
    from paper_conf_asplos_azamifb25_b200 import lcf_cpu
    lcf_cpu.lib()
    nt = os.cpu_count() or 1
    host = []
    for j in jobs:
        words = j["x"].cpu().numpy()
        host.append((j, words.view(np.uint32 if words.dtype == np.int32 else np.uint64),
                     j["s"][: j["sbytes"]].cpu().numpy()))
    total, spent, same = 0, 0.0, True
    for j, words, s_gpu in host:
        t0 = time.perf_counter()
        s = lcf_cpu.lcf_cpu_compress(j["codec"], words, n_threads=nt)
        y = lcf_cpu.lcf_cpu_decompress(j["codec"], s, n_threads=nt)
        spent += time.perf_counter() - t0
        total += 2 * words.nbytes
        same = same and s.tobytes() == s_gpu.tobytes() and np.array_equal(y, words)
    return {"value": total / spent / 1e9, "unit": "GB/s", "cores": nt, "kind": "cpu_codec (liblcf_cpu.so)",
            "streams_equal_gpu": bool(same),
            "sample": "whole CESM T/U and Miranda density/rt_density fields with their codecs, compress + decompress"}


def run_reference(args):
    """--impl reference: the CPU oracle as it stands, on rank 0 only."""
    world, rank, local = dist_env()
    if rank != 0:
        return
    import oracle
    from paper_conf_asplos_azamifb25_b200 import datagen
    oracle.lib()
    sample_bytes = 1 << 20
    cuda = torch.cuda.is_available()
    samples = []
    for cfg, names, codecs in FIELD_SETS:
        for nm in names:
            if cuda:  # the lcf arm's exact fields (generated on the device, as there)
                x = datagen.field(cfg, nm, device="cuda").reshape(-1)[: sample_bytes // 4].cpu()
            elif cfg.startswith("hacc"):  # (generated whole; a prefix of a shorter array of the same kind)
                x = datagen._hacc(nm, datagen._gen(datagen.seed_of(5, {"xx": 0, "vx": 1}[nm]), "cpu"), "cpu",
                                  (sample_bytes // 4,), None)
            else:  # the leading planes of the field, drawn on the host
                shape = datagen.CONFIGS[cfg][1]
                sub = (max(1, (sample_bytes // (4 if cfg.endswith("f32") else 8)) // (shape[-1] * (
                    shape[-2] if len(shape) == 3 else 1)) + 1),) + tuple(shape[1:])
                x = datagen.field(cfg, nm, device="cpu", origin=(0,) * len(shape), shape=sub)
            w = x.numpy().reshape(-1).view(np.uint32 if x.dtype == torch.float32 else np.uint64)
            w = w[: sample_bytes // w.itemsize].copy()
            for c in codecs:
                samples.append((c, w))
    times = []
    total = 0
    for it in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        total = 0
        for c, w in samples:
            s = oracle.compress(c, w)
            oracle.decompress(c, s)
            total += 2 * w.nbytes
        if it >= args.warmup:
            times.append(time.perf_counter() - t0)
    t = statistics.median(times)
    v = total / t / 1e9
    print(json.dumps({
        "impl": "reference", "metric": "compress+decompress throughput (uncompressed GB/s)", "value": v,
        "unit": "GB/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32/u64 (f32/f64 bits)",
        "data": "synthetic", "config": {"workload": WORKLOAD, "sample": "first 1 MiB of every (codec, field)",
                                        "l2": "n/a (host oracle)"},
        "cpu_baseline": {"value": v, "unit": "GB/s", "cores": 1, "kind": "oracle",
                         "sample": "first 1 MiB of every (codec, field) of the workload per step"},
        "e2e": {"value": v, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }))


def spawn_ranks(args) -> int:
    """`--gpus N` without a launcher: re-run this script under
    torch.distributed.run with N processes on this node (127.0.0.1), one per
    GPU; rank 0's JSON line is the output."""
    import socket
    sock = socket.socket()
    sock.bind(("127.0.0.1", 0))
    port = sock.getsockname()[1]
    sock.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def dry_run(args):
    """--dry-run: the multi-rank plumbing only (process group, rank layout,
    the max-over-ranks reduction) — no device work; gloo when there is no GPU."""
    import torch.distributed as dist
    world, rank, local = dist_env()
    if world > 1:
        dist.init_process_group("nccl" if torch.cuda.is_available() else "gloo")
    t = torch.tensor([float(rank + 1)])
    if world > 1 and not torch.cuda.is_available():
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    if rank == 0:
        print(json.dumps({"dry_run": True, "n_gpus": world, "max_over_ranks": float(t.item()),
                          "backend": dist.get_backend() if world > 1 else None}))
    if world > 1:
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="lcf", choices=["lcf", "reference"])
    ap.add_argument("--codecs", default=",".join(ALL_CODECS))
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-transfer", action="store_true",
                    help="N >= 2: skip the rank 0 -> rank 1 raw vs compressed NCCL transfer (transfer.py)")
    ap.add_argument("--dry-run", action="store_true", help="multi-rank plumbing only (tests)")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        if not args.dry_run and args.impl == "lcf" and torch.cuda.device_count() < args.gpus:
            sys.exit(f"bench.py --gpus {args.gpus}: only {torch.cuda.device_count()} CUDA devices visible")
        sys.exit(spawn_ranks(args))
    if world != args.gpus and not (args.impl == "reference" and world == 1):
        sys.exit(f"bench.py --gpus {args.gpus} launched with WORLD_SIZE={world}")
    args.transfer = not args.no_transfer
    if args.dry_run:
        dry_run(args)
    elif args.impl == "reference":
        run_reference(args)
    else:
        run_lcf(args)


if __name__ == "__main__":
    main()
