#!/usr/bin/env python
"""Benchmark of the LaSAGNA hot path on B200 (BASELINE.json metric: reads/s and overlap
edges/s, HBM GB/s vs peak).

One step = the whole hot path over the configured synthetic read set: 2-bit pack (a1) ->
fingerprints + key tables (a2/a3) -> LSD sort (a4) -> suffix search + verify (a5) -> greedy
claim (a6) -> succ/olen edge arrays (a7).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config cfg3] [--impl native|reference]

N > 1 runs under torchrun (one rank per GPU, NCCL): hash-range sharded tables, see
paper_conf_ipps_goswamilsp18_b200/dist.py.  Rank 0 prints ONE JSON line.
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

import readgen  # noqa: E402

METRIC = "reads/sec and overlap edges/sec at 1/2/4/8 B200; HBM GB/s vs peak"
DEFAULT_CONFIG = "cfg3"  # BASELINE configs[2]: the config the 1/2/4/8-GPU metric is quoted on


def _peaks() -> dict:
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return {"hbm_gbs": float(d["hbm_gbs"]), "source": "measured (MEASURED_PEAKS.json)"}
    except Exception:
        return {"hbm_gbs": 6650.0, "source": "fallback (B200_PROFILING.md)"}


# ------------------------------------------------------------------ clocks during the timed region
class ClockSampler:
    FIELDS = ["clocks.sm", "clocks.max.sm", "power.draw", "clocks_event_reasons.hw_slowdown",
              "clocks_event_reasons.hw_thermal_slowdown", "clocks_event_reasons.sw_thermal_slowdown",
              "clocks_event_reasons.sw_power_cap"]

    def __init__(self, bus_id: str | None):
        self.bus_id = bus_id
        self.lines: list[str] = []
        self.proc = None
        self.thread = None

    def start(self):
        cmd = ["nvidia-smi", "--query-gpu=" + ",".join(self.FIELDS), "--format=csv,noheader,nounits",
               "-lms", "200"]
        if self.bus_id:
            cmd[1:1] = ["-i", self.bus_id]
        try:
            self.proc = subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.DEVNULL,
                                         text=True)
        except (OSError, FileNotFoundError):
            self.proc = None
            return
        def rd():
            for line in self.proc.stdout:
                self.lines.append(line.strip())
        self.thread = threading.Thread(target=rd, daemon=True)
        self.thread.start()

    def stop(self) -> dict:
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in self.lines:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                smax.append(float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def _bus_id(torch, dev: int) -> str | None:
    try:
        p = torch.cuda.get_device_properties(dev)
        return f"{p.pci_domain_id:08X}:{p.pci_bus_id:02X}:{p.pci_device_id:02X}.0"
    except Exception:
        return None


# ------------------------------------------------------------------ CPU oracle baseline
def cpu_baseline(reads: np.ndarray, l_min: int, target_s: float = 12.0) -> dict:
    """The oracle as it stands, timed on a bounded prefix of the same read set."""
    import oracle
    cores = os.cpu_count() or 1
    os.environ.setdefault("OMP_NUM_THREADS", str(cores))
    oracle.lib()
    n_total = reads.shape[0]
    n0 = min(n_total, 50_000)
    t = time.perf_counter()
    oracle.greedy_graph(reads[:n0], l_min)
    t0 = time.perf_counter() - t
    n1 = int(min(n_total, max(n0, n0 * target_s / max(t0, 1e-3))))
    t = time.perf_counter()
    _, _, m, acc = oracle.greedy_graph(reads[:n1], l_min)
    t1 = time.perf_counter() - t
    return {"value": n1 / t1, "unit": "reads/s", "cores": int(os.environ["OMP_NUM_THREADS"]),
            "kind": "oracle",
            "sample": f"first {n1} reads of the workload (oracle.greedy_graph, exact-string "
                      f"overlaps + sequential greedy; {m} read-end pairs), {t1:.2f} s"}


# ------------------------------------------------------------------ algorithmic bytes
def roofline(stats: dict, n: int, L: int, l_min: int, steps: int, peak: dict,
             sm_mhz: float | None = None) -> dict:
    """Dominant phase and its achieved ALGORITHMIC GB/s (bytes per unit in DESIGN.md x units
    per launch / CUDA-event time per launch)."""
    V = 2 * n
    N = V                         # table entries per length (one canonical entry per vertex)
    n_len = L - l_min
    G = stats["lengths_per_pass"]
    verify = 64.0 * (stats["n_pairs"] + stats["fp_false_matches"]) / max(1, n_len)
    bucketed = bool(stats.get("bucketed", 1))
    if bucketed:
        per = {
            # level-1 partition fused with the fingerprints: every key written once
            "scatter_table_kernel": (stats["ms_table"], stats["passes"], 8.0 * G * N + 32.0 * n),
            # level-2 partition: every key read once and written once
            "refine_kernel": (stats["ms_sort"], stats["sort_launches"], 16.0 * G * N),
            # one join launch (one length): every key read once + verification loads
            "bucket_join_kernel": (stats["ms_search"], stats["search_launches"], 8.0 * N + verify),
        }
    else:
        per = {
            # one onesweep pass over a group: every key read once and written once
            "onesweep_kernel": (stats["ms_sort"], stats["sort_launches"], 16.0 * G * N),
            # one join launch (one length): the sorted table streamed once + verification loads
            "join_kernel": (stats["ms_search"], stats["search_launches"], 8.0 * N + verify),
            # table: 4 keys (32 B) written per read per length, the packed read loaded once
            "table_kernel": (stats["ms_table"], stats["passes"], 8.0 * G * N + 32.0 * n),
        }
    name = max(per, key=lambda k: per[k][0])
    ms, launches, bytes_per_launch = per[name]
    launches = max(1, launches)
    avg_s = ms / 1e3 / launches
    achieved = bytes_per_launch / avg_s / 1e9 if avg_s > 0 else 0.0
    traffic = None
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as f:
            traffic = json.load(f).get(name)
    except Exception:
        pass
    phases = {k: {"ms_per_step": v[0] / steps, "launches_per_step": v[1] / steps,
                  "gbs": (v[2] / (v[0] / 1e3 / max(1, v[1])) / 1e9) if v[0] > 0 else None}
              for k, v in per.items()}
    phases["greedy"] = {"ms_per_step": stats["ms_greedy"] / steps}
    # Issue view of the same kernel (integer-ALU-bound kernels): warp instructions per launch
    # from the committed ncu capture (profiles/ncu_inst.json) over the live launch time, against
    # the SM issue peak = SMs x 4 schedulers x 1 warp instruction per cycle x the SM clock.
    issue = None
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_inst.json")) as f:
            inst = json.load(f).get(name)
        if inst and avg_s > 0:
            import torch
            sms = torch.cuda.get_device_properties(0).multi_processor_count
            ghz = (sm_mhz or 1965.0) / 1e3
            pk = sms * 4 * ghz
            ach = inst / avg_s / 1e9
            issue = {"unit": "G warp-inst/s", "achieved": round(ach, 1), "peak": round(pk, 1),
                     "frac": round(ach / pk, 4), "inst_per_launch": inst,
                     "peak_basis": f"{sms} SMs x 4 issue/clk x {ghz:.3f} GHz (measured SM clock)"}
    except Exception:
        pass
    return {"bound": "hbm", "kernel": name, "achieved": round(achieved, 1),
            "peak": peak["hbm_gbs"], "peak_source": peak["source"], "unit": "GB/s",
            "frac": round(achieved / peak["hbm_gbs"], 4), "traffic": traffic,
            "bytes_per_launch": bytes_per_launch, "issue": issue, "phases": phases}


# ------------------------------------------------------------------ reference arm (the oracle)
def run_reference(args, cfg, rank: int) -> None:
    if rank != 0:
        return
    reads = readgen.config_reads(cfg, n=min(cfg.n, 4_000_000))
    import oracle
    cores = os.cpu_count() or 1
    os.environ.setdefault("OMP_NUM_THREADS", str(cores))
    oracle.lib()
    # bounded per-step sample: ~10 s of CPU work per step
    n0 = min(reads.shape[0], 50_000)
    t = time.perf_counter()
    oracle.greedy_graph(reads[:n0], cfg.l_min)
    t0 = time.perf_counter() - t
    ns = int(min(reads.shape[0], max(n0, n0 * 8.0 / max(t0, 1e-3))))
    for _ in range(args.warmup if args.warmup < 1 else 1):
        oracle.greedy_graph(reads[:ns], cfg.l_min)
    times, pairs = [], 0
    for _ in range(args.steps):
        t = time.perf_counter()
        _, _, pairs, _ = oracle.greedy_graph(reads[:ns], cfg.l_min)
        times.append(time.perf_counter() - t)
    tot = sum(times)
    value = ns * args.steps / tot
    out = {"metric": METRIC, "value": value, "unit": "reads/s", "n_gpus": args.gpus,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * tot / args.steps,
           "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u64",
           "data": "synthetic", "impl": "reference",
           "config": {"workload": f"{cfg.name}: {cfg.note}", "sample_reads": ns, "n": cfg.n,
                      "L": cfg.L, "l_min": cfg.l_min},
           "overlap_edges_per_s": 2 * pairs * args.steps / tot,
           "cpu_baseline": {"value": value, "unit": "reads/s",
                            "cores": int(os.environ["OMP_NUM_THREADS"]), "kind": "oracle",
                            "sample": f"first {ns} reads of {cfg.name} per step"},
           "e2e": {"value": value, "unit": "reads/s", "h2d_bytes_per_step": 0,
                   "d2h_bytes_per_step": 0},
           "gpu_launches": 0}
    print(json.dumps(out), flush=True)


# ------------------------------------------------------------------ native arm
def main() -> None:
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default=DEFAULT_CONFIG, choices=sorted(readgen.CONFIGS))
    ap.add_argument("--impl", default="native", choices=["native", "reference"])
    ap.add_argument("--lengths-per-pass", type=int, default=0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--n", type=int, default=0, help="override read count (debug)")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="process-group backend of the multi-GPU path (gloo: ranks may share a GPU)")
    ap.add_argument("--force-dist", action="store_true",
                    help="run the sharded multi-GPU path even with one rank")
    args = ap.parse_args()
    cfg = readgen.CONFIGS[args.config]
    if args.n:
        from dataclasses import replace
        cfg = replace(cfg, n=args.n)

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if args.impl == "reference":
        run_reference(args, cfg, rank)
        return
    if world > 1 or args.force_dist:
        from paper_conf_ipps_goswamilsp18_b200 import dist
        dist.bench_main(args, cfg, METRIC, _peaks(), ClockSampler, _bus_id, cpu_baseline)
        return

    import torch
    import paper_conf_ipps_goswamilsp18_b200 as lz
    assert args.warmup >= 3 or os.environ.get("BENCH_ALLOW_SHORT_WARMUP"), "W >= 3"
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    n, L, l_min = cfg.n, cfg.L, cfg.l_min
    # ---- synthetic reads straight into pinned host memory (generator time excluded)
    host = torch.empty((n, L), dtype=torch.uint8).pin_memory()
    readgen.reads_into(host.data_ptr(), cfg.seed, cfg.G, L, cfg.p_err, 0, n)
    dev_ascii = host.to(dev)  # device-resident input for `value`
    runner = lz.GreedyGraph(n, L, l_min, dev, args.lengths_per_pass)
    h_succ = torch.empty(2 * n, dtype=torch.int32).pin_memory()
    h_olen = torch.empty(2 * n, dtype=torch.uint8).pin_memory()
    stream = torch.cuda.current_stream(dev)

    def step(src, with_d2h: bool, stats: bool):
        # a1-a7 from the ASCII reads through the public API (staging fused into the first
        # table pass; from pinned host memory the PCIe read-in overlaps the fingerprints)
        r = runner.from_ascii(src, stats=stats)
        if with_d2h:
            h_succ.copy_(r.succ, non_blocking=True)
            h_olen.copy_(r.olen, non_blocking=True)
        return r

    for _ in range(args.warmup):
        r = step(dev_ascii, False, True)
    torch.cuda.synchronize()
    check_stats = r.stats

    # ---- device-resident timed region
    sampler = ClockSampler(_bus_id(torch, 0))
    agg = {k: 0.0 for k in ["ms_table", "ms_sort", "ms_search", "ms_greedy"]}
    cnt = {k: 0 for k in ["sort_launches", "search_launches", "passes"]}  # summed over steps
    sampler.start()
    torch.cuda.synchronize()
    launches0 = lz.kernel_launches()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(args.steps):
        r = step(dev_ascii, False, True)
        for k in agg:
            agg[k] += r.stats[k]
        for k in cnt:
            cnt[k] += r.stats[k]
    e1.record(stream)
    torch.cuda.synchronize()
    launches = lz.kernel_launches() - launches0
    clocks = sampler.stop()
    ms_total = e0.elapsed_time(e1)
    ms_step = ms_total / args.steps
    st = dict(r.stats)
    st.update(agg)
    st.update(cnt)
    value = n / (ms_step / 1e3)
    edges = 2 * st["n_pairs"]

    # ---- end to end through the public API: pinned host ASCII -> ... -> succ/olen on host.
    # (1) one batch at a time (latency): GreedyGraph.from_ascii on the page-locked input
    # (chunked DMA inside the call); (2) two batches in flight (throughput, the e2e value):
    # GraphPipeline — batch k+1's host -> device copy overlaps batch k's device work and
    # read-back.  Every step copies its whole input in and its whole result out.
    for _ in range(1):
        step(host, True, False)
    torch.cuda.synchronize()
    f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    f0.record(stream)
    for _ in range(args.steps):
        step(host, True, False)
    f1.record(stream)
    torch.cuda.synchronize()
    e2e_serial_ms = f0.elapsed_time(f1) / args.steps
    ref_succ = h_succ.numpy().copy()

    del dev_ascii, runner
    torch.cuda.empty_cache()
    pipe = lz.GraphPipeline(n, L, l_min, dev, args.lengths_per_pass)
    outs = [(torch.zeros(2 * n, dtype=torch.int32).pin_memory(),
             torch.empty(2 * n, dtype=torch.uint8).pin_memory()) for _ in range(2)]

    def pipelined(k_total: int) -> float:
        torch.cuda.synchronize()
        g0, g1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        g0.record(pipe.copy)
        for s_ in pipe.lanes:
            s_.wait_event(g0)
        pipe.run([host] * k_total, [outs[k % 2] for k in range(k_total)])
        for s_ in pipe.lanes:
            pipe.copy.wait_stream(s_)
        g1.record(pipe.copy)
        torch.cuda.synchronize()
        return g0.elapsed_time(g1)

    pipelined(2)  # warm-up of both runners
    e2e_ms = pipelined(args.steps) / args.steps
    for j in range(2):  # both in-flight lanes produced the serial result
        assert np.array_equal(outs[j][0].numpy(), ref_succ), f"lane {j} differs"

    peak = _peaks()
    roof = roofline(st, n, L, l_min, args.steps, peak, clocks.get("sm_mhz"))
    out = {
        "metric": METRIC, "value": value, "unit": "reads/s", "n_gpus": 1, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "u64", "data": "synthetic",
        "config": {"workload": f"{cfg.name}: {cfg.note}", "n": n, "L": L, "l_min": l_min,
                   "G": cfg.G, "p_err": cfg.p_err, "seed": cfg.seed,
                   "lengths_per_pass": st["lengths_per_pass"], "passes": st["passes"] // args.steps,
                   "l2": "inputs larger than L2 (ASCII %.1f GB, key tables %.1f GB)"
                         % (n * L / 1e9, 16.0 * 2 * n * st["lengths_per_pass"] / 1e9)},
        "overlap_edges_per_s": edges / (ms_step / 1e3),
        "read_end_pairs": st["n_pairs"], "greedy_pairs": st["n_greedy"],
        "fp_false_matches": st["fp_false_matches"], "greedy_rounds_max": st["rounds_max"],
        "e2e": {"value": n / (e2e_ms / 1e3), "unit": "reads/s", "ms_per_step": e2e_ms,
                "h2d_bytes_per_step": n * L, "d2h_bytes_per_step": 2 * n * 5,
                "batches_in_flight": 2, "serial_ms_per_step": e2e_serial_ms,
                "serial_value": n / (e2e_serial_ms / 1e3)},
        "roofline": roof,
        "clocks": clocks,
        "gpu_launches": launches,
    }
    if not args.no_cpu_baseline:
        out["cpu_baseline"] = cpu_baseline(host.numpy(), l_min)
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
