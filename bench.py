#!/usr/bin/env python
"""Benchmark of the ISP hot path (BASELINE.json configs[1]) on B200.

Step = one pass of the hot path over one batch: the 5x5 binomial Gaussian (f32) over a
4096 x 4096 image in all four border modes (Clamp, Mirror, Repeat, Constant), variant
AUTO ("isp+m": the Eq. (10) model picks ISP or naive), i.e. 4 kernel launches.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl {isp,reference}]

N = 1: the 4096^2 image.  N > 1 (torchrun, one rank per GPU, NCCL): weak scaling --
each rank owns a 4096-row strip of a (4096 N) x 4096 image and exchanges 2-row halos
with its neighbours (ring for Repeat) through isp_shard_filter_f32.
value = output pixels of all ranks / max-over-ranks time (Mpixel/s).

Timing: W untimed warm-up steps, then exactly K steps replayed from CUDA graphs
(one graph per rotation phase), bracketed by barrier + synchronize, timed with CUDA
events on the launch stream; inputs rotate over 6 in/out buffer pairs (768 MiB > 2x
L2), so every launch reads cold HBM.  nvidia-smi clocks are sampled during the timed
region.  --impl reference times the CPU oracle (oracle/, test infrastructure) on the
host cores over a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "Mpixel/s & HBM GB/s fraction per filter/border mode; ISP speedup vs naive"
UNIT = "Mpixel/s"
MODES = ["clamp", "mirror", "repeat", "constant"]
N_SIDE = 4096
WINDOW = 5
CONST = 0.5
NPAIRS = 6
BYTES_PER_PX = 8          # algorithmic: one f32 read + one f32 write per output pixel


def env_rank():
    return int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), int(os.environ.get("LOCAL_RANK", 0))


def gauss_mask():
    import synth
    b = synth.binomial_row(WINDOW).astype(np.float64)
    return (np.outer(b, b) / b.sum() ** 2).astype(np.float32)


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


def lib_digest():
    import hashlib
    try:
        h = hashlib.sha256(open(os.path.join(ROOT, "paper_conf_ipps_qiaoth21_b200", "libisp.so"), "rb").read())
        return h.hexdigest()[:16]
    except OSError:
        return None


def ncu_traffic(workload):
    """DRAM bytes (read + write) per launch of the dominant kernel, measured by ncu over a
    range of >= 8 back-to-back launches (so write-backs are counted) -- `ncu` replays
    kernels, so it cannot run inside this timed process; tools/ncu_traffic.py writes
    profiles/r<NN>_traffic_<workload>.json and records the libisp.so digest it measured.
    Returned with its source file and whether that digest matches the library loaded now."""
    import glob
    paths = sorted(glob.glob(os.path.join(ROOT, "profiles", f"r*_traffic_{workload}.json")))
    if not paths:
        return {"traffic": None, "traffic_source": None}
    try:
        d = json.load(open(paths[-1]))
    except Exception:
        return {"traffic": None, "traffic_source": None}
    return {"traffic": d.get("dram_bytes_per_launch"), "traffic_source": os.path.relpath(paths[-1], ROOT),
            "traffic_build_matches": d.get("libisp_sha16") == lib_digest(),
            "traffic_launches": d.get("launches")}


class ClockSampler:
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, device_index):
        self.dev = device_index
        self.proc = None
        self.path = os.path.join("/tmp", f"isp_clocks_{os.getpid()}.csv")

    def __enter__(self):
        try:
            self.f = open(self.path, "w")
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                          "-lms", "50", "-i", str(self.dev)], stdout=self.f,
                                         stderr=subprocess.DEVNULL)
            time.sleep(0.3)
        except Exception:
            self.proc = None
        return self

    def __exit__(self, *a):
        if self.proc is not None:
            time.sleep(0.1)
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
            self.f.close()

    def summary(self, t0, t1):
        if self.proc is None:
            return None
        rows = []
        for line in open(self.path):
            parts = [p.strip() for p in line.split(",")]
            if len(parts) < 9:
                continue
            try:
                rows.append((float(parts[1]), float(parts[2]), parts[5:9]))
            except ValueError:
                continue
        if not rows:
            return None
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for (_, _, r) in rows for k in range(4) if r[k].lower().startswith("active")})
        loaded = [c for (c, _, _) in rows]
        return {"sm_mhz": statistics.median(loaded), "sm_max_mhz": max(m for (_, m, _) in rows),
                "reasons": reasons, "samples": len(rows)}


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    import platform
    return platform.processor() or "unknown"


def _oracle_rows_rate(img, mask, modes, threads, target_s):
    """Oracle throughput (Mpixel/s) on a centred row band sized for ~target_s seconds."""
    import oracle
    H, W = img.shape
    t = time.perf_counter()
    for m in modes:
        oracle.filter_f64(img, mask, m, CONST, rows=(0, 2 * threads), threads=threads)
    dt = time.perf_counter() - t
    rows = int(max(threads, min(H, 2 * threads * target_s / max(dt, 1e-6))))
    rows -= rows % threads
    rows = max(rows, threads)
    y0 = (H - rows) // 2
    t = time.perf_counter()
    for m in modes:
        oracle.filter_f64(img, mask, m, CONST, rows=(y0, y0 + rows), threads=threads)
    dt = time.perf_counter() - t
    px = len(modes) * rows * W
    return px / dt / 1e6, f"rows [{y0},{y0 + rows}) x {len(modes)} modes ({px} px, {dt:.1f} s)", dt


def cpu_oracle_rate(target_s=8.0, threads=None, workload=None):
    """Oracle (oracle/ C, double accumulation, per-read border map) on the host cores over a
    bounded row sample of the same workload and modes: once on 1 thread and once on all
    cores.  `value` / `cores` are the all-core run."""
    import oracle
    import synth
    threads = threads or os.cpu_count() or 1
    oracle.build_oracle()
    if workload is None or workload.name == "cfg2":
        img = synth.uniform_f32(N_SIDE, N_SIDE, synth.CONFIG_SEEDS["cfg2"])
        mask, modes, name = gauss_mask(), MODES, "cfg2 4096x4096"
    else:   # cfg5: a 512-row band of the 16384-wide image is enough for the bounded sample
        img = synth.uniform_f32(512, workload.W, synth.CONFIG_SEEDS["cfg5"])
        mask, modes, name = workload.mask(), workload.modes, "cfg5 16384-wide (512-row band)"
    v1, s1, d1 = _oracle_rows_rate(img, mask, modes, 1, target_s / 2)
    vn, sn, dn = _oracle_rows_rate(img, mask, modes, threads, target_s)
    return {"value": vn, "unit": UNIT, "cores": threads, "kind": "oracle",
            "sample": f"{name} image, all cores: {sn}; 1 thread: {s1}",
            "single_thread": {"value": v1, "unit": UNIT, "cores": 1, "sample": s1, "seconds": d1},
            "cpu_model": cpu_model(), "seconds": dn + d1}


# ------------------------------------------------------------------------------------------
def run_reference(args):
    rank, world, _ = env_rank()
    if rank != 0:
        return
    import oracle
    import synth
    threads = os.cpu_count() or 1
    oracle.build_oracle()
    img = synth.uniform_f32(N_SIDE, N_SIDE, synth.CONFIG_SEEDS["cfg2"])
    mask = gauss_mask()
    # each step = a bounded sample (rows_per_step rows x 4 modes), sized so the run ends in minutes
    rows_per_step = 16 * threads  # 16 rows per host thread and mode: amortises the per-call setup
    times = []
    for k in range(args.warmup + args.steps):
        y0 = (k * rows_per_step) % (N_SIDE - rows_per_step)
        t = time.perf_counter()
        for m in MODES:
            oracle.filter_f64(img, mask, m, CONST, rows=(y0, y0 + rows_per_step), threads=threads)
        if k >= args.warmup:
            times.append(time.perf_counter() - t)
    tot = sum(times)
    px = 4 * rows_per_step * N_SIDE * args.steps
    val = px / tot / 1e6
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * tot / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": "cfg2: 5x5 binomial Gaussian f32 4096x4096, 4 border modes (oracle sample)",
                       "sample_rows_per_step": rows_per_step},
            "cpu_baseline": {"value": val, "unit": UNIT, "cores": threads, "kind": "oracle",
                             "sample": f"{rows_per_step} rows x 4096 px x 4 modes per step",
                             "cpu_model": cpu_model()},
            "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------------------------------
class Workload:
    """cfg2 (default, BASELINE.json configs[1]): 5x5 binomial f32, 4 border modes, 4096^2
    per rank -- N ranks = row strips of a (4096 N) x 4096 image (weak scaling).
    cfg5 (configs[4], the north-star scaling case): 7x7 binomial f32 on ONE 16384^2 image,
    Clamp and Repeat, row strips over N ranks (strong scaling)."""

    def __init__(self, name, world):
        self.name = name
        if name == "cfg2":
            self.W, self.H = N_SIDE, N_SIDE * world
            self.window, self.modes, self.scaling = WINDOW, MODES, "weak"
            self.seed = 2
            self.desc = ("cfg2: 5x5 binomial Gaussian f32 4096x4096 per rank, 4 border modes "
                         "(clamp, mirror, repeat, constant), variant auto (isp+m)")
        else:
            self.W = self.H = 16384
            self.window, self.modes, self.scaling = 7, ["clamp", "repeat"], "strong"
            self.seed = 5
            self.desc = ("cfg5: 7x7 binomial Gaussian f32 on one 16384x16384 image, clamp + repeat, "
                         "variant auto (isp+m)")
        self.halo = self.window // 2

    def mask(self):
        import synth
        b = synth.binomial_row(self.window).astype(np.float64)
        return (np.outer(b, b) / b.sum() ** 2).astype(np.float32)


def run_isp(args):
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_qiaoth21_b200 as isp
    import synth

    rank, world, local = env_rank()
    # ISP_BENCH_SAME_DEVICE=1 (test hook): every rank on cuda:0 with a gloo process group
    # and the peer path only -- the multi-rank code on a one-GPU box (CUDA IPC works between
    # processes on one device; NCCL does not take two ranks per device)
    same_dev = os.environ.get("ISP_BENCH_SAME_DEVICE") == "1" and world > 1
    if same_dev:
        local = 0
        args.halo = "peer"
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    rdev = torch.device("cpu") if same_dev else dev      # device of the reduction tensors
    if world > 1:
        if same_dev:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)
    isp.lib()
    wl = Workload(args.workload, world)
    mask = wl.mask()
    modes = wl.modes
    nm = len(modes)
    H_img, W = wl.H, wl.W
    halo = wl.halo
    y0, sh = isp.isp_shard_rows(H_img, rank, world) if world > 1 else (0, H_img)
    # ---- inputs: seeded, resident in HBM before the timed region ----
    if wl.name == "cfg2":
        host_img = synth.uniform_f32(N_SIDE, N_SIDE, synth.CONFIG_SEEDS["cfg2"] + rank)
        src = torch.from_numpy(host_img)
    else:
        g = torch.Generator().manual_seed(wl.seed * 1000 + rank)
        src = torch.rand((sh, W), generator=g)
        host_img = None
    img_bytes = 2 * 4 * sh * W                       # one in + one out buffer
    npairs = NPAIRS if wl.name == "cfg2" else int(min(6, max(2, -(-2 * 126 * 2 ** 20 // img_bytes))))
    pairs = []
    for _ in range(npairs):
        if world > 1:
            strip = torch.empty((sh + 2 * halo, W), dtype=torch.float32, device=dev)
            strip[halo:halo + sh].copy_(src)
            inp = strip
        else:
            inp = src.to(dev)
        out = torch.empty((sh, W), dtype=torch.float32, device=dev)
        pairs.append((inp, out))
    ctx = None
    comm_stream = torch.cuda.Stream(device=dev)
    if world > 1 and not same_dev:
        uid = [isp.isp_shard_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(uid, src=0)
        ctx = isp.isp_shard_init(uid[0], rank, world, local)
    stream = torch.cuda.Stream(device=dev)
    variant = args.variant
    # N > 1 halo path: "peer" (default) -- every rank reads its neighbours' edge rows straight
    # from their strips over NVLink (CUDA IPC), one launch per rank and mode, no exchange;
    # "nccl" -- halo rows exchanged with NCCL send/recv, then the edge rows launched.
    halo_path = args.halo if world > 1 else None
    peers = None
    if world > 1 and halo_path == "peer":
        try:
            own = [pairs[k][0][halo:halo + sh] for k in range(npairs)]
            peers = []
            for o in own:   # CUDA IPC handles of every rank's strip, exchanged over the process group
                hs = [None] * world
                dist.all_gather_object(hs, isp.isp_shard_peer_handle(o))
                peers.append(isp.isp_shard_peer_attach(rank, world, o, hs, ring=True))
            ok = torch.tensor([1.0], device=rdev)
        except Exception as e:   # no IPC in this environment: fall back to the NCCL exchange
            print(f"[bench] rank {rank}: peer open failed ({e}); using the NCCL halo exchange", file=sys.stderr)
            ok = torch.tensor([0.0], device=rdev)
        dist.all_reduce(ok, op=dist.ReduceOp.MIN)
        if ok.item() < 1:
            if peers:
                for pp in peers:
                    isp.isp_shard_peer_close(pp)
            peers, halo_path = None, "nccl (peer open failed)"
        torch.cuda.synchronize()
        dist.barrier()      # every strip holds its data before any rank reads a neighbour's

    def launch(mode, pair, v=variant):
        inp, out = pairs[pair]
        if world > 1 and peers is not None:
            isp.isp_shard_peer_filter_f32(peers[pair], H_img, mask, mode, CONST, out=out, variant=v, stream=stream)
        elif world > 1:
            isp.isp_shard_filter_f32(ctx, inp, H_img, halo, mask, mode, CONST, out=out, variant=v, stream=stream,
                                     comm_stream=comm_stream)
        else:
            isp.isp_filter_ex(inp, mask, mode, CONST, out=out, variant=v, stream=stream)

    def step(k, v=variant):
        for i, m in enumerate(modes):
            launch(m, (nm * k + i) % npairs, v)

    if world > 1 and peers is not None:
        launches_per_step = nm
    elif world > 1:
        launches_per_step = sum(len([l for l in isp.isp_shard_schedule(H_img, rank, world, halo, halo,
                                                                       isp.MODES[m])["launch"] if l[1] > 0])
                                for m in modes)
    else:
        launches_per_step = nm
    nphase = npairs // int(np.gcd(nm, npairs))      # rotation period in steps
    use_graph = not args.no_graph

    with torch.cuda.stream(stream):
        for k in range(max(args.warmup, 1)):      # warm-up (also loads every kernel)
            step(k)
    torch.cuda.synchronize()
    # The timed region replays ONE graph holding exactly K steps (all launches back to
    # back, no inter-graph gaps); above MAX_GRAPH_STEPS steps it is a chunk graph of
    # MAX_GRAPH_STEPS steps replayed, plus one graph for the remainder.
    MAX_GRAPH_STEPS = 2000
    chunk_graph, rem_graph, n_chunks = None, None, 0

    def capture(nsteps, k0):
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=stream):
            for k in range(k0, k0 + nsteps):
                step(k)
        return g

    if use_graph:
        try:
            chunk = min(args.steps, MAX_GRAPH_STEPS)
            chunk -= chunk % nphase if args.steps > MAX_GRAPH_STEPS else 0
            n_chunks = args.steps // chunk
            chunk_graph = capture(chunk, 0)
            rem = args.steps - n_chunks * chunk
            rem_graph = capture(rem, n_chunks * chunk) if rem else None
            for g in (chunk_graph, rem_graph):
                if g is not None:
                    g.replay()
            torch.cuda.synchronize()
        except Exception as e:  # pragma: no cover
            print(f"[bench] graph capture failed ({e}); eager launches", file=sys.stderr)
            chunk_graph, rem_graph = None, None
            use_graph = False

    def run_steps(K, v=variant):
        """Exactly K steps (K == args.steps when graphs are used)."""
        with torch.cuda.stream(stream):
            if use_graph and v == variant and K == args.steps:
                for _ in range(n_chunks):
                    chunk_graph.replay()
                if rem_graph is not None:
                    rem_graph.replay()
            else:
                for k in range(K):
                    step(k, v)

    plan = isp.isp_last_plan()
    # ---- timed region ----
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as cs:
        t_wall0 = time.time()
        # keep the GPU busy (~2 ms spin, before the start event) while the host enqueues
        # the start event, the K-step graph and the stop event: the timed region is then
        # exactly the K steps on the device, not the host's graph-launch latency
        with torch.cuda.stream(stream):
            torch.cuda._sleep(4_000_000)
        e0.record(stream)
        run_steps(args.steps)
        e1.record(stream)
        torch.cuda.synchronize()
        t_wall1 = time.time()
    if world > 1:
        dist.barrier()
    ms = e0.elapsed_time(e1)
    if world > 1:
        t = torch.tensor([ms], device=rdev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    clocks = cs.summary(t_wall0, t_wall1)
    px_step = nm * H_img * W                 # output pixels of all ranks per step
    value = px_step * args.steps / (ms / 1e3) / 1e6
    ms_step = ms / args.steps

    # ---- per-launch duration of the dominant kernel (the ISP stencil) on this rank ----
    per_launch_us = 1e3 * ms_step / nm
    pk = peaks()
    hbm = pk.get("hbm_gbs")
    rank_bytes = BYTES_PER_PX * sh * W
    achieved = rank_bytes / (per_launch_us * 1e-6) / 1e9
    kname = f"OpSepF32<{wl.window},{wl.window}>"
    roof = {"bound": "hbm", "achieved": achieved, "peak": hbm if hbm else 6650.0, "unit": "GB/s",
            "frac": achieved / (hbm if hbm else 6650.0),
            "peak_source": "MEASURED_PEAKS.json hbm_gbs (measured)" if hbm else "fallback (B200_PROFILING.md)",
            "kernel": f"variant {args.variant}: " + (
                (f"k_sep_band<{wl.window}> (warp-strip band ISP, cp.async ring; band_f32.cu)" if plan["tile_w"] == 128
                 else f"k_pstaged<{kname}> (persistent TMA-staged ISP)" if os.environ.get("ISP_TMA_PERSIST") == "1"
                 else f"k_staged<{kname}> (TMA-staged ISP)") if plan["choice"] == 4 else f"k_stencil<{kname}>"),
            "algorithmic_bytes_per_launch": rank_bytes,
            "duration_us": per_launch_us,
            "duration_method": "timed region / launches (one CUDA graph of the K steps, kernels back to back)"}
    roof.update(ncu_traffic(wl.name))

    # ---- ISP vs naive per mode (same methodology, single-GPU variants) ----
    variants = {}
    if world == 1 and not args.quick:
        for m in modes:
            variants[m] = {}
            for v in ["auto", "tma", "warp", "block", "naive"]:
                R = 12 if wl.name == "cfg2" else 4
                g = torch.cuda.CUDAGraph()
                with torch.cuda.stream(stream):
                    for i in range(2):
                        launch(m, i % npairs, v)
                torch.cuda.synchronize()
                with torch.cuda.graph(g, stream=stream):
                    for i in range(R):
                        launch(m, i % npairs, v)
                torch.cuda.synchronize()
                reps = 40 if wl.name == "cfg2" else 5
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                with torch.cuda.stream(stream):
                    g.replay()
                    torch.cuda._sleep(2_000_000)
                    a.record(stream)
                    for _ in range(reps):
                        g.replay()
                    b.record(stream)
                torch.cuda.synchronize()
                us = 1e3 * a.elapsed_time(b) / (reps * R)
                variants[m][v] = {"us": us, "gbs": BYTES_PER_PX * H_img * W / (us * 1e-6) / 1e9,
                                  "mpix_s": H_img * W / us}
            for v in ("tma", "warp", "auto"):
                variants[m][f"speedup_{v}_vs_naive"] = variants[m]["naive"]["us"] / variants[m][v]["us"]

    # ---- halo exchange alone (N > 1): NCCL send/recv of the strip edges on the comm stream ----
    halo_us = None
    if world > 1 and ctx is not None:
        inp = pairs[0][0]
        R = 50
        dist.barrier()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(comm_stream):
            a.record(comm_stream)
            for _ in range(R):
                isp.isp_shard_exchange(ctx, inp, H_img, halo, halo, modes[-1], comm_stream=comm_stream)
            b.record(comm_stream)
        torch.cuda.synchronize()
        t = torch.tensor([a.elapsed_time(b) * 1e3 / R], device=rdev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        halo_us = float(t.item())

    # ---- end to end: pinned host buffers, H2D + filter + D2H inside the timed region ----
    e2e = None
    if not args.quick and not same_dev:
        hin = (torch.from_numpy(host_img) if host_img is not None else src).pin_memory()
        houts = [torch.empty((sh, W), dtype=torch.float32).pin_memory() for _ in range(2)]
        E = max(6, min(20, args.steps // 100)) if wl.name == "cfg2" else 3
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        if world > 1:
            with torch.cuda.stream(stream):
                a.record(stream)
                for k in range(E):
                    for i, m in enumerate(modes):
                        inp, out = pairs[i % npairs]
                        inp[halo:halo + sh].copy_(hin, non_blocking=True)
                        isp.isp_shard_filter_f32(ctx, inp, H_img, halo, mask, m, CONST, out=out, stream=stream,
                                                 comm_stream=comm_stream)
                        houts[i % 2].copy_(out, non_blocking=True)
                b.record(stream)
        else:
            # a user's pipeline: H2D, filter and D2H on three streams, launch j's upload
            # overlapping launch j-1's filter and launch j-2's download (PCIe is full duplex);
            # a device buffer pair is reused only after its previous filter / download finished
            s_in, s_out = torch.cuda.Stream(), torch.cuda.Stream()
            h2d_done, cmp_done, d2h_done = [], [], []
            a.record(s_in)
            j = 0
            for k in range(E):
                for i, m in enumerate(modes):
                    inp, out = pairs[j % npairs]
                    ev_in, ev_cmp, ev_out = torch.cuda.Event(), torch.cuda.Event(), torch.cuda.Event()
                    if j >= npairs:
                        s_in.wait_event(cmp_done[j - npairs])
                    with torch.cuda.stream(s_in):
                        inp.copy_(hin, non_blocking=True)
                    ev_in.record(s_in)
                    stream.wait_event(ev_in)
                    if j >= npairs:
                        stream.wait_event(d2h_done[j - npairs])
                    isp.isp_filter(inp, mask, m, CONST, out=out, stream=stream)
                    ev_cmp.record(stream)
                    s_out.wait_event(ev_cmp)
                    with torch.cuda.stream(s_out):
                        houts[j % 2].copy_(out, non_blocking=True)
                    ev_out.record(s_out)
                    h2d_done.append(ev_in)
                    cmp_done.append(ev_cmp)
                    d2h_done.append(ev_out)
                    j += 1
            b.record(s_out)
        torch.cuda.synchronize()
        ems = a.elapsed_time(b)
        if world > 1:
            t = torch.tensor([ems], device=rdev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ems = float(t.item())
        e2e = {"value": px_step * E / (ems / 1e3) / 1e6, "unit": UNIT,
               "h2d_bytes_per_step": nm * 4 * sh * W, "d2h_bytes_per_step": nm * 4 * sh * W,
               "steps": E, "ms_per_step": ems / E,
               "api": "isp_filter / isp_shard_filter_f32 via the Python binding, pinned host buffers; "
                      + ("H2D / filter / D2H pipelined on three streams" if world == 1 else "one stream")}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        cpu = cpu_oracle_rate(workload=wl)

    if peers is not None:
        torch.cuda.synchronize()
        dist.barrier()
        for pp in peers:
            isp.isp_shard_peer_close(pp)
    if ctx is not None:
        torch.cuda.synchronize()
        isp.isp_shard_destroy(ctx)
    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": wl.scaling,
                "vs_baseline": None, "dtype": "f32", "data": "synthetic",
                "config": {"workload": wl.desc
                                       + (f"; {world} ranks = row strips of the {H_img}x{W} image, halo rows "
                                          f"via {halo_path}" if world > 1 else ""),
                           "image": [H_img, W], "window": [wl.window, wl.window], "const": CONST,
                           "modes": modes,
                           "l2": f"rotating {npairs} in/out buffer pairs "
                                 f"({npairs * img_bytes // 2 ** 20} MiB per rank > 2x L2)",
                           "parallelism": f"row-strips x{world}" if world > 1 else "single GPU",
                           "cuda_graphs": use_graph, "plan": {k: plan[k] for k in
                                                              ("tile_w", "tile_h", "nx", "ny", "choice", "g",
                                                               "degenerate")}},
                "roofline": roof, "cpu_baseline": cpu, "e2e": e2e,
                "gpu_launches": args.steps * launches_per_step, "clocks": clocks,
                "isp_vs_naive": variants or None}
        if world > 1:
            line["halo_path"] = halo_path
            line["halo_exchange_us"] = halo_us
            line["per_rank_rows"] = sh
            line["config"]["halo"] = halo_path
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def check_launch(args):
    """--check-launch: the multi-rank launch path without a workload -- every rank joins
    the process group (NCCL on GPUs, gloo on a CPU box), all-reduces its rank id, rank 0
    prints what it saw.  Used by tests/test_bench_launch.py on CPU."""
    import torch
    import torch.distributed as dist
    rank, world, local = env_rank()
    backend = "nccl" if torch.cuda.is_available() else "gloo"
    if world > 1:
        if backend == "nccl":
            torch.cuda.set_device(local)
            dist.init_process_group(backend, device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    t = torch.tensor([float(rank)], device="cuda" if backend == "nccl" else "cpu")
    n = torch.ones(1, device=t.device)
    if world > 1:
        dist.all_reduce(t)
        dist.all_reduce(n)
    if rank == 0:
        print(json.dumps({"check": "launch", "world_size": world, "gpus_requested": args.gpus, "backend": backend,
                          "ranks_seen": int(n.item()), "rank_sum": int(t.item())}), flush=True)
    if world > 1:
        dist.destroy_process_group()


def spawn_ranks(args):
    """`bench.py --gpus N` started without torchrun: re-exec under torch.distributed.run with
    N ranks on this node (rendezvous on 127.0.0.1), as the driver does."""
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    env = dict(os.environ)
    env.setdefault("NCCL_DEBUG", "INFO")          # NCCL's init lines (nranks) stay visible
    env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd, env=env)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--workload", default="cfg2", choices=["cfg2", "cfg5"],
                    help="cfg2: BASELINE configs[1] (default, weak scaling over ranks); "
                         "cfg5: configs[4] 16384^2 7x7 strong scaling")
    ap.add_argument("--check-launch", action="store_true", help="only check the N-rank launch path")
    ap.add_argument("--halo", default="peer", choices=["peer", "nccl"],
                    help="N > 1: neighbour rows read from peer memory (default) or exchanged with NCCL")
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=20)
    ap.add_argument("--impl", default="isp", choices=["isp", "reference"])
    ap.add_argument("--variant", default="auto", choices=["auto", "tma", "warp", "block", "naive"])
    ap.add_argument("--no-graph", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--quick", action="store_true", help="skip the variant table and e2e (profiling runs)")
    args = ap.parse_args()
    if args.warmup < 3:
        ap.error("--warmup must be >= 3")
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(spawn_ranks(args))
    world = int(os.environ.get("WORLD_SIZE", 1))
    if world != args.gpus:
        ap.error(f"--gpus {args.gpus} but WORLD_SIZE={world}")
    if args.check_launch:
        check_launch(args)
        return
    if args.impl == "reference":
        run_reference(args)
    else:
        run_isp(args)


if __name__ == "__main__":
    main()
