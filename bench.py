#!/usr/bin/env python
"""Benchmark of the B200 MDMC skycube (BASELINE.json metric: "skycube build time & dominance tests/s,
n=1M d=12 anticorr, 1/2/4/8 B200").

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config H] [--impl ours|reference]
    python -m torch.distributed.run --nproc-per-node N --master-addr 127.0.0.1 ... bench.py --gpus N

`--gpus N` without torchrun re-launches itself as N ranks under torch.distributed.run (one process per GPU).

One step = one whole skycube build (K0 validate -> key sort -> K2 codes -> K1 prefilter -> S+ ->
K3 MDMC -> K4 compaction into membership rows and the per-subspace id lists) over the synthetic
workload, input resident in HBM.  value = dominance tests/s = n_ext*(n_ext-1) / (step time, max over
ranks).  e2e = the same metric through the C-ABI skycube_build_ex with host buffers (H2D of the
points and D2H of every output inside the timed region; N>1: host input -> per-rank pipeline ->
rank-0 D2H).  --impl reference times the CPU oracle (oracle/, the reference arm of this tier) on a
bounded sample of tasks, extrapolated to the whole build.
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

import datagen  # noqa: E402

METRIC = "skycube build time & dominance tests/s, n=1M d=12 anticorr, 1/2/4/8 B200"
UNIT = "dominance tests/s"
L2_FLUSH_BYTES = 256 << 20


def algorithmic_ops_per_test(d: int) -> int:
    """DESIGN.md §5 Roofline: one test of K3 (a chunk-corner test or a pair test) forms the d-bit mask
    B_{code<=code} (one compare per dimension: d) and probes B_{p notin S+} (one load + one bit test: 2)."""
    return d + 2


INTPEAK = os.path.join(ROOT, "profiles", "r02_intpeak.json")


def int_peaks(sm_mhz: float, sms: int = 148):
    """Integer lane-op peaks at the SM clock of the run, from the MEASURED microbenchmark
    (tools/intpeak.cu on one B200, profiles/r02_intpeak.json): lane-ops per SM per clock of (a) the ALU pipe
    alone (LOP3/IADD3/PRMT/SHF chains) and (b) ALU + FMA pipes together (LOP3 interleaved with IMAD, the
    one-warp-instruction-per-SMSP-per-clock issue bound).  Falls back to the B300_MICROARCH pipe rates
    (rt_SMSP = 2 per pipe: 64 and 128 lanes/SM/clk) only if the measurement file is absent, and says so."""
    try:
        with open(INTPEAK) as f:
            m = json.load(f)
        alu = m["alu"]["lane_ops_per_sm_per_clk"]
        mix = max(m[k]["lane_ops_per_sm_per_clk"] for k in ("mix", "mix2") if k in m)
        basis = (f"measured (profiles/r02_intpeak.json: {alu:.1f} ALU-only and {mix:.1f} ALU+FMA integer lane-ops "
                 f"per SM per clock) x {sms} SMs x {sm_mhz:.0f} MHz (median SM clock of this run)")
    except Exception:
        alu, mix = 64.0, 128.0
        basis = f"FALLBACK (no profiles/r02_intpeak.json): B300_MICROARCH pipe rates 64 / 128 lanes/SM/clk x {sms} x {sm_mhz:.0f} MHz"
    return alu * sms * sm_mhz * 1e6, mix * sms * sm_mhz * 1e6, basis


def golden_fullsize(config: str):
    """The offline full-size Oracle B record of a config (tests/golden/fullsize_digests.json, written by
    tools/oracle_digest.py, which calls only oracle/), or None."""
    try:
        with open(os.path.join(ROOT, "tests", "golden", "fullsize_digests.json")) as f:
            return json.load(f)["configs"].get(config)
    except Exception:
        return None


def cpu_model() -> str:
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.startswith("Model name:"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def config_dict(cfg, args, world: int, m: int, total_ids) -> dict:
    """The `config` object of both arms (identical keys, so the driver can match them)."""
    return {"workload": workload(cfg), "n": cfg.n, "d": cfg.d, "n_ext": m, "pairs": m * (m - 1),
            "total_ids": total_ids, "output": args.output, "max_level": args.max_level or cfg.d,
            "l2": "256 MB buffer written between timed steps",
            "parallelism": (f"dp{world}: K1 tiles and K3 task groups sharded, S+ flags all-reduced, "
                            f"rows all-gathered" if world > 1 else "dp1")}


def ncu_traffic(config: str, kernel: str):
    """dram__bytes_read.sum + dram__bytes_write.sum of one launch of `kernel` at `config`, from the committed
    ncu --set full capture summarised in profiles/traffic.json (None if there is no capture)."""
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            t = json.load(f)
        e = t[config][kernel]
        return int(e["dram_read_bytes"]) + int(e["dram_write_bytes"]), e.get("source")
    except Exception:
        return None, None


def ncu_instructions(config: str, kernel: str):
    """smsp__inst_executed.sum (warp instructions) of one launch of `kernel` at `config` and the tests the
    same launch executed (device counters), from the committed ncu capture summarised in profiles/traffic.json."""
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            e = json.load(f)[config][kernel]
        if "warp_instructions" in e and "tests" in e:
            return e
    except Exception:
        pass
    return None


def workload(cfg) -> str:
    return f"{cfg.name}: {cfg.dist} n={cfg.n} d={cfg.d} seed={cfg.seed} (datagen, Börzsönyi-style)"


def env_rank():
    return int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")), int(os.environ.get("LOCAL_RANK", "0"))


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled every 200 ms during the timed region."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int, path: str | None = None):
        self.index = index
        self.proc = None
        self.path = path

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None
        time.sleep(0.3)
        return self

    def __exit__(self, *a):
        self.lines = []
        if self.proc is not None:
            self.proc.terminate()
            try:
                out, _ = self.proc.communicate(timeout=5)
            except Exception:
                self.proc.kill()
                out = ""
            self.lines = [l for l in out.splitlines() if l.strip()]
            if self.path:
                with open(self.path, "w") as f:
                    f.write("\n".join(self.lines) + "\n")

    def summary(self):
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for l in getattr(self, "lines", []):
            parts = [p.strip() for p in l.split(",")]
            if len(parts) < 9:
                continue
            try:
                sm.append(float(parts[1]))
                mx = float(parts[2])
            except ValueError:
                continue
            for nm, v in zip(names, parts[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        loaded = [s for s in sm if mx and s > 0.5 * mx] or sm
        return {"sm_mhz": statistics.median(loaded) if loaded else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="H", choices=sorted(datagen.CONFIGS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--clocks-log", default=None)
    ap.add_argument("--output", default="lattice", choices=["lattice", "hashcube", "both"],
                    help="skycube representation built by each step: the lattice (K4, Fig. 1a, default), the "
                         "HashCube (K5, w=32, Alg. 3 line 13 / Fig. 1b) or both")
    ap.add_argument("--max-level", type=int, default=0, help="partial skycube d' (Appendix A.2); 0 = full")
    ap.add_argument("--algo", default="mdmc", choices=["mdmc", "sdsc"],
                    help="mdmc (the product path, default) or the SDSC comparator (Alg. 2, skycube_build_sdsc; "
                         "1 GPU, host buffers, timed end to end)")
    return ap.parse_args()


# ------------------------------------------------------------------------------ CPU oracle timing
def oracle_sample_time(x: np.ndarray, target_s: float, seed: int = 0):
    """Time Oracle B on a seeded uniform sample of tasks (per-task work is independent of the others,
    so time * n / sample extrapolates the full build).  Returns (seconds for the whole build,
    sample size, seconds measured, estimated n_ext, threads)."""
    import oracle
    n = x.shape[0]
    rng = np.random.default_rng(seed)
    k = 8
    t = 0.0
    while True:
        pids = rng.choice(n, size=min(k, n), replace=False)
        t0 = time.perf_counter()
        rows, ext = oracle.rows_b(x, pids, with_ext=True)
        t = time.perf_counter() - t0
        if t >= target_s / 4 or k >= n:
            break
        k = min(n, int(k * max(2.0, (target_s / 4) / max(t, 1e-3))))
    full_bit = (1 << x.shape[1]) - 1
    in_ext = ((ext[:, full_bit >> 5] >> (full_bit & 31)) & 1).astype(bool)
    est_next = int(round(in_ext.mean() * n))
    return t * n / len(pids), len(pids), t, est_next, oracle.num_threads()


def run_reference(args):
    rank, world, _ = env_rank()
    if rank != 0:
        return
    cfg = datagen.config(args.config)
    x = cfg.data()
    per_step = max(2.0, min(20.0, 150.0 / max(1, args.steps + args.warmup)))
    times = []
    for i in range(args.warmup + args.steps):
        full_s, k, t, est_next, thr = oracle_sample_time(x, per_step, seed=i)
        if i >= args.warmup:
            times.append((full_s, k, t, est_next, thr))
    full = statistics.median([a[0] for a in times])
    gold = golden_fullsize(args.config)
    if gold is not None and not args.max_level:
        # exact |S+| and id count of this workload, computed offline by the oracle itself (tools/oracle_digest.py)
        m, total_ids, m_src = gold["n_ext"], gold["total_ids"], "exact (tests/golden/fullsize_digests.json, Oracle B)"
    else:
        m, total_ids, m_src = times[0][3], None, "estimated from the sample's S+ bits"
    value = m * (m - 1) / full
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": full * 1e3, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": config_dict(cfg, args, args.gpus, m, total_ids),
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": times[0][4], "kind": "oracle",
                         "cpu_model": cpu_model(),
                         "sample": f"Oracle B (oracle/skycube_oracle.c, -O2) rows for {times[0][1]} uniformly sampled "
                                   f"points of {cfg.n} per step ({times[0][2]:.1f} s on {times[0][4]} threads), "
                                   f"extrapolated x n/sample; n_ext {m_src}"},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    if gold is not None:
        o = gold["oracle"]
        line["cpu_baseline"]["full_run"] = (f"the whole workload was run once by tools/oracle_digest.py: Oracle B over all "
                                            f"{cfg.n} points in {o['rows_b_wall_s']:.0f} s on {o['threads']} threads "
                                            f"({o['cpu_model']}, -O3 -march=native build of the same source)")
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------------------ GPU arm
def run_ours(args):
    import torch
    import torch.distributed as dist

    from paper_conf_sigmod_boghcsa17_b200 import build as skybuild
    rank, world, local = env_rank()
    if world > 1 and not dist.is_initialized():
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    torch.cuda.set_device(local)
    if rank == 0:
        skybuild.build()
    if world > 1:
        dist.barrier()
    import paper_conf_sigmod_boghcsa17_b200 as sky
    from paper_conf_sigmod_boghcsa17_b200.pipeline import DeviceSkycube

    cfg = datagen.config(args.config)
    x = cfg.data()
    n, d = x.shape
    dev = torch.device("cuda", local)
    pts = torch.from_numpy(x).to(dev)
    flush = torch.empty(L2_FLUSH_BYTES // 4, dtype=torch.int32, device=dev)
    eng = DeviceSkycube(local)
    names = ["t0", "t1", "t2", "t3", "t4"]

    lists = args.output in ("lattice", "both")
    hc_w = 32 if args.output in ("hashcube", "both") else 0

    def step(events=None):
        return eng.build(pts, lists=lists, membership=True, events=events, hashcube_w=hc_w,
                         max_level=args.max_level)

    out = None
    for _ in range(args.warmup):
        out = step()
    if out is None:  # --warmup 0 (profiling runs): one untimed build still fixes n_ext and the id count
        out = step()
    torch.cuda.synchronize()
    m = out["n_ext"]
    total_ids = out.get("total_ids", 0)
    hc_ids = int(out["hashcube"]["ids"].numel()) if hc_w else None
    ev = [{k: torch.cuda.Event(enable_timing=True) for k in names} for _ in range(args.steps)]
    launches0 = eng.launches
    cnt0 = eng.ctx.counters()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local, args.clocks_log) as clk:
        t_start = torch.cuda.Event(enable_timing=True)
        t_end = torch.cuda.Event(enable_timing=True)
        t_start.record()
        for s in range(args.steps):
            flush.fill_(s)  # L2 flush between steps (256 MB > 126 MB L2)
            step(ev[s])
        t_end.record()
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    launches = eng.launches - launches0
    cnt1 = eng.ctx.counters()
    work = {k: (cnt1[k] - cnt0[k]) / args.steps for k in cnt1}
    step_ms = [ev[s]["t0"].elapsed_time(ev[s]["t4"]) for s in range(args.steps)]
    phase = {k: statistics.mean(ev[s][a].elapsed_time(ev[s][b]) for s in range(args.steps))
             for k, a, b in [("prepare", "t0", "t1"), ("prefilter", "t1", "t2"), ("mdmc", "t2", "t3"),
                             ("compact", "t3", "t4")]}
    total_ms = sum(step_ms)
    if world > 1:
        tt = torch.tensor([total_ms, phase["mdmc"]], dtype=torch.float64, device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        total_ms, mdmc_max = tt.tolist()
    ms_per_step = total_ms / args.steps
    pairs = m * (m - 1)
    value = pairs / (ms_per_step / 1e3)

    # ---- e2e through the public API with host buffers
    e2e = None
    if not args.no_e2e:
        e2e = measure_e2e(args, x, eng, world, rank, dev, pairs)

    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    if rank != 0:
        return
    clocks = clk.summary()
    sm_mhz = clocks["sm_mhz"] or 1965.0
    # roofline of the dominant kernel (K3 MDMC), duration from CUDA events on its stream; its work is
    # the tests it must run after static-tree pruning (device counters), not the n_ext^2 pairs it resolves
    mdmc_ms = phase["mdmc"]
    tests = work["k3_box"] + work.get("k3_sub", 0) + work["k3_pair"]
    ops = tests * algorithmic_ops_per_test(d)
    achieved = ops / (mdmc_ms / 1e3) / 1e12
    peak_alu, peak_mix, peak_basis = int_peaks(sm_mhz)
    peak = peak_mix / 1e12
    traffic, traffic_src = ncu_traffic(args.config, "k3_mdmc") if world == 1 else (None, None)
    conf = config_dict(cfg, args, world, m, total_ids)
    if hc_w:
        conf["output"] += f" (w=32, {hc_ids} stored ids)"
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": conf,
        "phases_ms": phase,
        "work_per_step": work,
        "gpu_launches": launches,
        "roofline": {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "Tlane-op/s",
                     "frac": achieved / peak, "frac_alu_only": achieved / (peak_alu / 1e12),
                     "traffic": traffic, "traffic_unit": "bytes (DRAM read+write per launch)",
                     "traffic_source": traffic_src,
                     "kernel": "k3_mdmc", "ops_per_test": algorithmic_ops_per_test(d), "tests": tests,
                     "resolved_pairs": pairs,
                     "peak_basis": "peak = ALU+FMA integer issue bound; frac_alu_only against the ALU pipe alone; "
                                   + peak_basis},
        "clocks": clocks,
    }
    ins = ncu_instructions(args.config, "k3_mdmc") if world == 1 else None
    if ins:
        line["roofline"]["ncu_lane_instructions_per_test"] = 32.0 * ins["warp_instructions"] / ins["tests"]
        line["roofline"]["ncu_lane_instructions_per_resolved_pair"] = 32.0 * ins["warp_instructions"] / pairs
        line["roofline"]["ncu_alu_pipe_pct"] = ins.get("alu_pipe_pct")
        line["roofline"]["ncu_source"] = ins.get("source")
    if e2e is not None:
        line["e2e"] = e2e
    if not args.no_cpu and world == 1 or (not args.no_cpu and rank == 0 and world == 1):
        full_s, k, t, est_next, thr = oracle_sample_time(x, args.cpu_seconds)
        cpu_value = pairs / full_s
        line["cpu_baseline"] = {"value": cpu_value, "unit": UNIT, "cores": thr, "kind": "oracle",
                                "cpu_model": cpu_model(),
                                "sample": f"Oracle B rows for {k} uniformly sampled points of {n} "
                                          f"({t:.1f} s on {thr} threads), extrapolated x n/sample to "
                                          f"{full_s:.0f} s for the whole build"}
    print(json.dumps(line), flush=True)


def measure_e2e(args, x, eng, world, rank, dev, pairs):
    import torch
    import torch.distributed as dist
    n, d = x.shape
    if world == 1:
        import paper_conf_sigmod_boghcsa17_b200 as sky
        # the step's input sits in pinned host memory (the contract's e2e: pinned H2D inside the timed region)
        x_pinned = torch.from_numpy(np.ascontiguousarray(x, dtype=np.float32)).pin_memory()
        x = x_pinned.numpy()
        if args.output == "hashcube":
            def call():
                return sky.skycube_build_hashcube_raw(x, 32, stats=True, max_level=args.max_level)

            def d2h_bytes(r):
                a = r.arrays()
                return sum(int(v.nbytes) for v in a.values())
            api = "skycube_build_hashcube (C-ABI, host buffers, pinned result pool)"
        else:
            def call():
                return sky.skycube_build_raw(x, stats=True, lists=args.output != "hashcube", max_level=args.max_level)

            def d2h_bytes(r):
                return 4 * r.n_ext + 4 * n * sky.words_per_row(d) + 8 * ((1 << d) + 1) + 4 * int(r.offsets()[-1])
            api = "skycube_build_ex (C-ABI, host buffers, pinned result pool)"
        r = call()  # warm (pinned pools, contexts)
        d2h = d2h_bytes(r)
        r.close()
        times, phases = [], []
        for _ in range(args.e2e_steps):
            t0 = time.perf_counter()
            r = call()
            times.append(time.perf_counter() - t0)
            phases.append(r.stats)
            r.close()
        t = statistics.median(times)
        keys = ("ms_h2d", "ms_sort", "ms_prefilter", "ms_mdmc", "ms_compact", "ms_d2h", "ms_total")
        return {"value": pairs / t, "unit": UNIT, "h2d_bytes_per_step": int(x.nbytes), "d2h_bytes_per_step": int(d2h),
                "ms_per_step": t * 1e3, "api": api, "calls": len(times),
                "note": "median of the calls; the result buffers come from the library's pinned pool (allocated by the "
                        "warm-up call, reused after)",
                "phases_ms": {k: statistics.median(p[k] for p in phases) for k in keys}}
    # N > 1: pinned host input -> every rank H2D -> sharded pipeline; every rank writes its own membership rows
    # (and the zero rows of its id slice) and its lattice segments straight into pinned host buffers (zero-copy
    # over its own PCIe link); rank 0 also copies offsets and ext_ids.  The result is distributed over the ranks'
    # host buffers (global positions); d2h bytes are summed over the ranks.
    host = torch.from_numpy(x).pin_memory()
    W = (1 << d) >> 5 if d >= 5 else 1
    warm = eng.build(host.to(dev), lists=True, membership=False)
    total = warm["total_ids"]
    h_mem = torch.empty((n, W), dtype=torch.int32).pin_memory()
    h_ids = torch.empty(max(total, 1), dtype=torch.int32).pin_memory()
    times = []
    d2h = 0
    for i in range(args.e2e_steps + 1):
        dist.barrier()
        t0 = time.perf_counter()
        pts = host.to(dev, non_blocking=True)
        out = eng.build(pts, lists=True, membership=False, out_membership=h_mem, out_ids=h_ids)
        extra = []
        if rank == 0:
            extra = [out["offsets"].cpu(), out["ext_ids"].cpu()]
        torch.cuda.synchronize()
        dist.barrier()
        if i:
            times.append(time.perf_counter() - t0)
        else:
            j0, j1 = out["shard"]
            lo, hi = n * rank // world, n * (rank + 1) // world
            ext = out["ext_ids"].cpu().numpy()
            non_ext_in_slice = (hi - lo) - int(((ext >= lo) & (ext < hi)).sum())
            # membership rows this rank writes (its tasks + the non-S+ rows of its id slice) and its copies; the
            # lattice ids are written exactly once over all ranks (4 * total)
            mine = (j1 - j0 + non_ext_in_slice) * W * 4 + sum(t.numel() * t.element_size() for t in extra)
            d2h_t = torch.tensor([mine], dtype=torch.int64, device=dev)
            dist.all_reduce(d2h_t)
            d2h = int(d2h_t.item()) + 4 * total
    t = statistics.median(times)
    return {"value": pairs / t, "unit": UNIT, "h2d_bytes_per_step": int(x.nbytes) * world, "d2h_bytes_per_step": int(d2h),
            "ms_per_step": t * 1e3, "calls": len(times),
            "api": ("pipeline.DeviceSkycube (per-rank C-ABI device entry points; every rank writes its rows and "
                    "lattice segments zero-copy into pinned host buffers)")}


def run_sdsc(args):
    """The SDSC comparator (Alg. 2) on the same workload through its C-ABI call (host buffers, H2D and D2H
    inside the timed region); reported as its own JSON line with "algo": "sdsc"."""
    import paper_conf_sigmod_boghcsa17_b200 as sky
    from paper_conf_sigmod_boghcsa17_b200 import build as skybuild
    skybuild.build()
    cfg = datagen.config(args.config)
    x = cfg.data()
    n, d = x.shape
    r = sky.skycube_build_sdsc(x, stats=True)  # warm
    m = r["n_ext"]
    times, st = [], []
    for _ in range(max(1, args.steps)):
        t0 = time.perf_counter()
        r = sky.skycube_build_sdsc(x, stats=True)
        times.append(time.perf_counter() - t0)
        st.append(r["stats"])
    t = statistics.median(times)
    pairs = m * (m - 1)
    print(json.dumps({
        "algo": "sdsc", "metric": METRIC, "value": pairs / t, "unit": UNIT, "n_gpus": 1, "steps": len(times),
        "warmup": 1, "ms_per_step": t * 1e3, "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
        "dtype": "u32", "data": "synthetic",
        "config": {"workload": workload(cfg), "n": n, "d": d, "n_ext": m, "total_ids": int(r["offsets"][-1])},
        "phases_ms": {k: statistics.median(s[k] for s in st) for k in ("ms_h2d", "ms_sort", "ms_prefilter", "ms_mdmc", "ms_d2h")},
        "note": "ms_mdmc is the SDSC lattice traversal (Alg. 2 lines 2-7)"}), flush=True)


def spawn_ranks(args) -> int:
    """`bench.py --gpus N` without a torchrun environment: re-launch this script as N ranks (one process per
    GPU) under torch.distributed.run on 127.0.0.1, with NCCL_DEBUG=INFO so the communicator lines show the N
    ranks.  The ranks' JSON line (rank 0) goes to stdout; every other line of theirs to stderr."""
    import socket
    import torch
    have = torch.cuda.device_count()
    if have < args.gpus:
        sys.stderr.write(f"bench.py: --gpus {args.gpus} requested but only {have} CUDA device(s) are visible\n")
        return 2
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
    env = dict(os.environ)
    env.setdefault("NCCL_DEBUG", "INFO")
    env.setdefault("OMP_NUM_THREADS", "4")
    proc = subprocess.Popen(cmd, env=env, stdout=subprocess.PIPE, text=True, bufsize=1)
    for line in proc.stdout:
        (sys.stdout if line.lstrip().startswith("{") else sys.stderr).write(line)
        sys.stdout.flush()
    return proc.wait()


def main():
    args = parse()
    if args.gpus > 1 and "LOCAL_RANK" not in os.environ and args.impl == "ours" and args.algo == "mdmc":
        sys.exit(spawn_ranks(args))
    if "WORLD_SIZE" in os.environ and args.gpus > 1 and int(os.environ["WORLD_SIZE"]) != args.gpus:
        sys.exit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={os.environ['WORLD_SIZE']}")
    if args.algo == "sdsc":
        run_sdsc(args)
        return
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
