"""Benchmark of the community-reordered CSR SpMV hot path (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl reference]
                    [--config 5] [--orderings original,rabbit,rabbitpp]
                    [--exchange coll|peer]

Default workload, every N: BASELINE.json configs[4] -- power iteration on the
Graph500 Kronecker scale-28 graph (268 M rows, 4.26 G nnz, int64 row
pointers), row-block partitioned across the N GPUs, the largest
configuration in BASELINE.json and the one its "1/2/4/8 B200" metric scales
over.  A step is one power-iteration step of spmv_iterate (PAPER.md:221
"SpMV iterations"; reading c22): the scaled SpMV y = B u / s over this rank's
rows with the fixed-order sum of y^2, the all-reduce of that sum and the
exchange of the y slices (N > 1).  K steps run as one spmv_iterate call,
bracketed by a barrier + device synchronisation and timed with CUDA events on
the launching stream; max over ranks.  B and x are resident in HBM; the
matrix (37.8 GB) and x (1.07 GB) are far larger than the 126 MB L2, so no
flush is needed between steps.

value = ideal bytes of one SpMV of the whole matrix (PAPER.md:96 with the
real offset width) / step time, in GB/s, whole job; runtime / ideal =
peak / value (peak = measured copy bandwidth).

Input preparation is reported separately (PAPER.md:221 amortisation): the
matrix is generated on the GPU (synth.config_gpu, the host generator's exact
CSR), rank 0 reorders on the host (RABBIT / RABBIT++ with concurrent merges,
SURVEY §8(f4)) and broadcasts the permutation, every rank builds its plan and
B = P A P^T on its GPU.

Configs 1-4 (--config k) time one plain spmv_exec per step with the L2
flushed (a 512 MiB read and a reset of the persisting L2 lines) before every
step, outside the events.

--impl reference: the oracle (plain C fp64 CSR loop, oracle/c) timed on the
host cores on a bounded sample of the same reordered workload.
scripts/suite.py runs every config and the geometric mean of runtime / ideal.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "SpMV runtime & DRAM bytes ÷ ideal, achieved HBM GB/s, GFLOP/s at 1/2/4/8 B200"
FALLBACK_HBM = 6650.0
L2_BYTES = 126 * 2**20
NCU_SUMMARY = os.path.join("profiles", "ncu_summary.json")


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json)"
    return FALLBACK_HBM, "fallback (B200_PROFILING.md)"


class Clocks:
    """nvidia-smi sampler for the timed region."""

    def __init__(self, index=0):
        self.index, self.samples, self.proc = index, [], None

    def start(self):
        q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            parts = [s.strip() for s in line.split(",")]
            if len(parts) >= 7:
                self.samples.append(parts)

    def stop(self):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
        sms = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for s in self.samples for i in range(4)
                          if s[3 + i].lower().startswith("active")})
        return {"sm_mhz": statistics.median(sms) if sms else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": reasons,
                "samples": len(self.samples)}


def host_info():
    """CPU model and core count of this host (lscpu), for cpu_baseline."""
    model = None
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for ln in out.splitlines():
            if ln.startswith("Model name:"):
                model = ln.split(":", 1)[1].strip()
    except Exception:
        pass
    return {"model": model, "logical_cpus": os.cpu_count()}


def ncu_traffic(workload: str, ordering: str):
    p = os.path.join(ROOT, NCU_SUMMARY)
    if not os.path.exists(p):
        return None
    d = json.load(open(p))
    e = d.get(f"{workload}/{ordering}")
    return e if isinstance(e, dict) else None


GATHER_CEILING = os.path.join("profiles", "r67_gather_ceiling.jsonl")


def gather_ceiling():
    """Measured random 4-byte LDG gathers per second on this GPU type, x range
    L2-resident (scripts/gather_ceiling.cu, r67): the L1TEX rate of one 128-B
    line per clock per SM that a gather touching its own line costs."""
    p = os.path.join(ROOT, GATHER_CEILING)
    if not os.path.exists(p):
        return None
    best = 0.0
    for ln in open(p):
        d = json.loads(ln)
        if d.get("mode") == "ldg" and d.get("range_mb", 1e9) <= 64:
            best = max(best, float(d["ggather_per_s"]))
    return best * 1e9 if best else None


def ideal_bytes(n, nnz):
    """PAPER.md:96 with the real row-offset width (reading c2)."""
    return 2 * n * 4 + (n + 1) * (8 if nnz >= 2**31 else 4) + 2 * nnz * 4


# ------------------------------------------------------------------ inputs
class Inputs:
    """The workload on this rank's device: row_ptr / col / val tensors, host x,
    host pattern (rank 0, for the reorder), generator timing."""

    def __init__(self, k, dev, need_host: bool, small: bool = False):
        import numpy as np
        import torch

        import synth
        t = time.perf_counter()
        self.k = k
        if k in (1, 3, 5):   # RMAT / Kronecker: generated on the GPU
            self.name, A, self.x = synth.config_gpu(k, device=dev.index or 0, small=small)
            self.n, self.nnz = A.n, A.nnz
            self.rp_d, self.col_d, self.val_d = A.row_ptr, A.col, A.val
            # the reorder needs the pattern only; values come to the host later
            # (cpu_baseline), so the host never holds two copies at its peak
            self.host = synth.Csr(A.n, A.row_ptr.cpu().numpy(), A.col.cpu().numpy(), None) \
                if need_host else None
            self.where = "gpu (synth_gpu, bit-identical to the host generator)"
        else:
            w = synth.config(k, small=small)
            self.name, self.x, A = w.name, w.x, w.A
            self.n, self.nnz = A.n, A.nnz
            self.rp_d = torch.from_numpy(A.row_ptr).to(dev)
            self.col_d = torch.from_numpy(A.col).to(dev)
            self.val_d = torch.from_numpy(A.val).to(dev)
            self.host = A
            self.where = "host (synth)"
        if self.nnz < 2**31:
            self.rp_d = self.rp_d.to(torch.int32)
        torch.cuda.synchronize(dev)
        self.gen_s = time.perf_counter() - t
        self.x = np.ascontiguousarray(self.x, np.float32)


def reorder(args, inp, ordering):
    """spmv_reorder on the host (rank 0); --perm-cache memoises for dev runs."""
    import numpy as np
    from paper_conf_ispass_balajicjk23_b200 import spmv
    if args.perm_cache:
        f = os.path.join(args.perm_cache, f"{inp.name}_{ordering}_{args.seed}.npz")
        if os.path.exists(f):
            d = np.load(f, allow_pickle=True)
            return d["perm"], d["stats"].item()
    perm, st = spmv.reorder(inp.host.row_ptr, inp.host.col, ordering, seed=args.seed,
                            parallel=ordering not in ("original", "random", "degsort")
                            and not args.sequential_reorder)
    st = dict(st.__dict__)
    if args.perm_cache:
        os.makedirs(args.perm_cache, exist_ok=True)
        np.savez(f, perm=perm, stats=np.array(st, dtype=object))
    return perm, st


def share_perm(perm, n, dev, world, rank):
    """Rank 0's permutation to every rank (NCCL broadcast of the device copy)."""
    import torch
    import torch.distributed as dist
    if rank == 0:
        pd = torch.from_numpy(perm).to(dev)
    else:
        pd = torch.empty(n, dtype=torch.int32, device=dev)
    if world > 1:
        dist.broadcast(pd, src=0)
    return pd


# --------------------------------------------------------------------- GPU
def run_gpu(args):
    import numpy as np
    import torch
    import torch.distributed as dist

    from paper_conf_ispass_balajicjk23_b200 import dist as pdist, spmv

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.single_device:  # test mode: every rank on cuda:0 (gloo only)
        local = 0
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        if args.backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(args.backend)
    iterate_mode = args.config == 5
    inp = Inputs(args.config, dev, need_host=rank == 0, small=args.small)
    hbm, peak_src = peaks()
    ideal = ideal_bytes(inp.n, inp.nnz)
    orderings = args.orderings.split(",")
    main = orderings[-1]
    stream = torch.cuda.Stream(device=dev)   # non-legacy: the L2 window is a stream attribute
    torch.cuda.set_stream(stream)
    flush = None
    if not iterate_mode:
        flush = torch.zeros(512 * 2**20 // 4, dtype=torch.float32, device=dev)
        sink = torch.zeros((), dtype=torch.float32, device=dev)
        lib = spmv.lib()

    def flush_l2():
        # a 512 MiB read evicts normal lines; persisting lines (the plan's
        # access-policy window on x_B[0:H)) need an explicit reset
        torch.sum(flush, dim=0, out=sink)
        lib.spmv_reset_persisting_l2(None)

    comm = None
    if world > 1 and args.backend == "nccl":
        comm = pdist.nccl_comm_ptr(device=dev)
    results, line, main_info = {}, None, None
    for ordering in orderings:
        if rank == 0:
            t = time.perf_counter()
            perm, st = reorder(args, inp, ordering)
            st["wall_s"] = time.perf_counter() - t
        else:
            perm, st = None, {}
        if world > 1:
            dist.barrier()
        perm_d = share_perm(perm, inp.n, dev, world, rank)
        torch.cuda.synchronize(dev)
        t0 = time.perf_counter()
        P = spmv.Plan(inp.rp_d, inp.col_d, inp.val_d, perm_d, world=world, rank=rank,
                      variant=args.variant, nccl_comm=comm, permute=False,
                      exchange=spmv.EXCHANGE_PEER if args.exchange == "peer" else spmv.EXCHANGE_COLL)
        torch.cuda.synchronize(dev)
        plan_s = time.perf_counter() - t0
        # B = P A P^T timed on its own: algorithmic bytes
        # 16 NZ + 20 N (read A, gather perm, write B, row pointers, inv)
        pe0, pe1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        pe0.record(stream)
        P.permute(stream)
        pe1.record(stream)
        torch.cuda.synchronize(dev)
        permute_ms = pe0.elapsed_time(pe1)
        nnz_loc = P.info()["nnz_local"]
        permute_bytes = 16 * nnz_loc + 20 * (P.info()["row_end"] - P.info()["row_begin"])
        info = P.info()
        hc = pb = None
        if world > 1 and args.backend != "nccl":
            hc = pdist.HostColl(device=dev)
            P.set_coll(hc.coll)
        if world > 1 and args.exchange == "peer":
            pb = pdist.PeerBuffers(P, dev)
        x_d = torch.from_numpy(inp.x).to(dev)
        xB = P.permute_vec(x_d)
        is_main = ordering == main
        K = args.steps if is_main else max(5, args.steps // 4)
        y = torch.empty(max(info["row_end"] - info["row_begin"], 1), dtype=torch.float32, device=dev)
        if iterate_mode:
            xs = xB.clone()
            launches_per_step = info["exec_launches"] + 2   # + the fixed-order norm (2 kernels)

            def warm(w):
                P.iterate(xs, w)

            def timed(k):
                P.iterate(xs, k)
        else:
            launches_per_step = info["exec_launches"]

            def warm(w):
                for _ in range(w):
                    flush_l2()
                    P.exec(xB, y)
        warm(args.warmup)
        torch.cuda.synchronize(dev)
        clocks = Clocks(local) if is_main and rank == 0 else None
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize(dev)
        if clocks:
            clocks.start()
            time.sleep(0.3)
        wall0 = time.perf_counter()
        if iterate_mode:
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            timed(K)
            e1.record(stream)
            torch.cuda.synchronize(dev)
            times = [e0.elapsed_time(e1) / K]
        else:
            ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                  for _ in range(K)]
            for i in range(K):
                flush_l2()
                ev[i][0].record(stream)
                P.exec(xB, y)
                ev[i][1].record(stream)
            torch.cuda.synchronize(dev)
            times = [a.elapsed_time(b) for a, b in ev]
        wall = time.perf_counter() - wall0
        if world > 1:
            dist.barrier()
        ck = clocks.stop() if clocks else None
        ms = sum(times) / len(times)
        if world > 1:
            t = torch.tensor([ms], dtype=torch.float64, device=dev)
            if args.backend == "nccl":
                dist.all_reduce(t, op=dist.ReduceOp.MAX)
            else:
                h = t.cpu()
                dist.all_reduce(h, op=dist.ReduceOp.MAX)
                t.copy_(h)
            ms = float(t.item())
        gbs = ideal / (ms * 1e-3) / 1e9
        res = {"ms": ms, "gbs_ideal_over_t": gbs, "gflops": 2 * inp.nnz / (ms * 1e-3) / 1e9,
               "runtime_over_ideal": hbm / gbs, "reorder_s": st.get("seconds"),
               "plan_s": plan_s, "permute_ms": permute_ms,
               "permute_gbs": permute_bytes / (permute_ms * 1e-3) / 1e9,
               "H": info["hot_prefix"], "cta_rows": info["n_cta_rows"],
               "mid_rows": info["n_mid_rows"], "hub_rows": info["n_hub_rows"],
               "l2_window_bytes": P.info()["l2_window_bytes"],
               "stream_evict_first": info["stream_evict_first"]}
        if not iterate_mode:
            res["ms_median"] = statistics.median(times)
        for f in ("insularity", "insular_frac", "n_communities", "largest_comm_frac",
                  "modularity", "skew", "n_hubs", "parallel", "n_deferred", "seconds_detect"):
            if f in st:
                res[f] = st[f]
        if world > 1:
            b = P.export_partition()
            res["partition_rows"] = [b[k + 1] - b[k] for k in range(world)]
        if world == 1 and not args.no_side and not iterate_mode:
            res["spmm4"] = side_measure("spmm4", P, inp, info, K, flush_l2, stream, dev, hbm)
            res["coo"] = side_measure("coo", P, inp, info, K, flush_l2, stream, dev, hbm)
        tr = ncu_traffic(inp.name, ordering)
        if tr:
            res["dram_over_ideal_ncu"] = tr.get("dram_bytes", 0) / ideal
        results[ordering] = res
        if is_main:
            main_info = dict(info)
            if iterate_mode:
                e2e = e2e_iterate(P, inp, perm_d, args, dev, ideal, world, rank)
            else:
                e2e = e2e_exec(P, inp, args, dev, ideal)
            line = dict(metric=METRIC, value=round(gbs, 2), unit="GB/s", n_gpus=world, steps=K,
                        warmup=args.warmup, ms_per_step=round(ms, 5), higher_is_better=True,
                        scaling="strong", vs_baseline=None, dtype="f32", data="synthetic")
            line["config"] = {
                "workload": f"{inp.name} (BASELINE configs[{args.config - 1}])",
                "n": inp.n, "nnz": inp.nnz, "ordering": ordering,
                "parallelism": f"row-block x{world}" if world > 1 else "1 GPU",
                "step": ("spmv_iterate power-iteration step: exec_scaled over this rank's rows + "
                         "fixed-order sum y^2" + (" + all-reduce + " + (
                             "peer-store exchange (PEER)" if args.exchange == "peer" else
                             "all-gatherv (grouped ncclBroadcast)") if world > 1 else ""))
                if iterate_mode else "spmv_exec",
                "l2": ("inputs larger than L2 (matrix %.1f GB, x %.2f GB vs 126 MB): no flush"
                       % (ideal / 1e9, 4 * inp.n / 1e9)) if iterate_mode else
                      "flushed before every step (512 MiB read + persisting-L2 reset, outside the events)",
                "ideal_bytes": ideal,
                "ideal_bytes_paper_4B_offsets": 2 * inp.n * 4 + (inp.n + 1 + 2 * inp.nnz) * 4,
                "generator": inp.where,
                "kernel_variant": ["lane", "panel"][args.variant],
                "wall_s_timed_region": round(wall, 4)}
            line["runtime_over_ideal"] = round(hbm / gbs, 4)
            line["gflops"] = round(2 * inp.nnz / (ms * 1e-3) / 1e9, 2)
            line["roofline"] = {
                "bound": "hbm", "achieved": round(gbs, 2), "peak": hbm, "unit": "GB/s",
                "frac": round(gbs / hbm, 4),
                "traffic": tr.get("dram_bytes") if tr else None,
                "traffic_measured_in_run": False,
                "traffic_source": NCU_SUMMARY if tr else None,
                "kernel": "the SpMV of a step: k_lane + k_warp_rows + k_cta_rows + k_hub_chunk/"
                          "k_hub_fix on three streams (one launch sequence per step)",
                "peak_source": peak_src,
                "algorithmic_bytes_per_launch": ideal}
            gc = gather_ceiling()
            if gc:
                # the step gathers x once per entry; an L2-resident gather that
                # touches its own 128-B line costs one L1TEX wavefront, so
                # nnz / ceiling is the step's floor unless lanes share lines
                floor_ms = inp.nnz / gc * 1e3
                line["gather_roofline"] = {
                    "bound": "l1tex wavefronts of the x gathers", "gathers_per_step": inp.nnz,
                    "ceiling_gathers_per_s": round(gc), "floor_ms": round(floor_ms, 4),
                    "frac": round(floor_ms / ms, 4), "measured_in_run": False,
                    "source": GATHER_CEILING + " (scripts/gather_ceiling.cu, random 4-B LDG, "
                                               "L2-resident range, 4-16 in flight)"}
            line["e2e"] = e2e
            line["gpu_launches"] = launches_per_step * K + (1 if iterate_mode else 0)
            line["clocks"] = ck
            line["input_prep"] = {"generate_s": round(inp.gen_s, 3),
                                  "reorder_s": round(st.get("wall_s", 0.0), 3) if rank == 0 else None,
                                  "plan_s": round(plan_s, 4), "permute_ms": round(permute_ms, 3),
                                  "permute_gbs": round(permute_bytes / (permute_ms * 1e-3) / 1e9, 1),
                                  "permute_bytes_algorithmic": permute_bytes}
        if pb is not None:
            pb.close()
        P.close()
    line["orderings"] = {k: {kk: (round(vv, 5) if isinstance(vv, float) else vv)
                             for kk, vv in v.items()} for k, v in results.items()}
    base = results.get("random") or results.get("original")
    if base and main in results and rank == 0:
        saving = base["ms"] - results[main]["ms"]
        rs = results[main].get("reorder_s") or 0.0
        line["amortization_iters_vs_" + ("random" if "random" in results else "original")] = \
            (rs * 1e3 / saving) if saving > 0 else None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        perm, _ = reorder(args, inp, main)
        line["cpu_baseline"] = cpu_baseline(inp, perm, budget_s=args.cpu_budget)
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def side_measure(kind, P, inp, info, K, flush_l2, stream, dev, hbm):
    """Table IV kernels on the same plan, cold L2 like the
    SpMV steps, ideal traffic "updated according to the kernel":
      spmm4: 8 NZ + (N+1) w_off + 16 N (X) + 16 N (Y)
      coo:   12 NZ + 4 N (x) + 4 N (y)"""
    import torch
    n, nnz = inp.n, inp.nnz
    if kind == "spmm4":
        X = torch.empty((n, 4), dtype=torch.float32, device=dev).uniform_(-1, 1)
        Y = torch.empty_like(X)
        ideal = 32 * n + (n + 1) * info["offset_bytes"] + 8 * nnz
        flops = 8 * nnz

        def run():
            P.exec_spmm4(X, Y)
    else:
        X = torch.empty(n, dtype=torch.float32, device=dev).uniform_(-1, 1)
        Y = torch.empty_like(X)
        ideal = 8 * n + 12 * nnz
        flops = 2 * nnz

        def run():
            P.exec_coo(X, Y)
    for _ in range(3):
        flush_l2()
        run()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(K)]
    torch.cuda.synchronize()
    for i in range(K):
        flush_l2()
        ev[i][0].record(stream)
        run()
        ev[i][1].record(stream)
    torch.cuda.synchronize()
    ms = sum(a.elapsed_time(b) for a, b in ev) / K
    gbs = ideal / (ms * 1e-3) / 1e9
    return {"ms": round(ms, 5), "ideal_bytes": ideal, "gbs_ideal_over_t": round(gbs, 2),
            "runtime_over_ideal": round(hbm / gbs, 4), "gflops": round(flops / (ms * 1e-3) / 1e9, 2)}


def e2e_exec(P, inp, args, dev, ideal):
    """Same metric through the public API with HOST buffers: pinned H2D of x,
    P x, exec, P^T y, D2H of y -- all inside the timed region.  Steps are
    software-pipelined over two buffer slots on three streams (H2D copy engine,
    compute, D2H copy engine), as a serving loop would run it."""
    import torch
    n = inp.n
    comp = torch.cuda.current_stream()
    s_in, s_out = torch.cuda.Stream(), torch.cuda.Stream()
    xh = torch.from_numpy(inp.x).pin_memory()
    yh = [torch.empty(n, dtype=torch.float32).pin_memory() for _ in range(2)]
    xd = [torch.empty(n, dtype=torch.float32, device=dev) for _ in range(2)]
    yd = [torch.empty(n, dtype=torch.float32, device=dev) for _ in range(2)]
    xB = torch.empty(n, dtype=torch.float32, device=dev)
    yB = torch.empty_like(xB)
    ev = {k: [torch.cuda.Event() for _ in range(2)] for k in ("h2d", "comp", "d2h")}
    started = [False, False]

    def step(i):
        b = i & 1
        if started[b]:
            s_in.wait_event(ev["comp"][b])
        with torch.cuda.stream(s_in):
            xd[b].copy_(xh, non_blocking=True)
        ev["h2d"][b].record(s_in)
        comp.wait_event(ev["h2d"][b])
        if started[b]:
            comp.wait_event(ev["d2h"][b])
        P.permute_vec(xd[b], out=xB)
        P.exec(xB, yB)
        P.permute_vec(yB, inverse=True, out=yd[b])
        ev["comp"][b].record(comp)
        s_out.wait_event(ev["comp"][b])
        with torch.cuda.stream(s_out):
            yh[b].copy_(yd[b], non_blocking=True)
        ev["d2h"][b].record(s_out)
        started[b] = True

    for i in range(args.warmup):
        step(i)
    torch.cuda.synchronize()
    K = args.steps
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(comp)
    s_in.wait_event(e0)
    for i in range(K):
        step(i)
    comp.wait_stream(s_out)
    e1.record(comp)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / K
    xd[0].copy_(xh)
    P.permute_vec(xd[0], out=xB)
    P.exec(xB, yB)
    P.permute_vec(yB, inverse=True, out=yd[0])
    if not torch.equal(yd[0].cpu(), yh[(K - 1) & 1]):
        raise RuntimeError("e2e: pipelined result differs from a direct call")
    return {"value": round(ideal / (ms * 1e-3) / 1e9, 2), "unit": "GB/s", "ms_per_step": round(ms, 5),
            "h2d_bytes_per_step": 4 * n, "d2h_bytes_per_step": 4 * n,
            "path": "pinned H2D x -> spmv_permute_vec -> spmv_exec -> spmv_permute_vec^T -> D2H y "
                    "(two slots, copy engines overlapped with the kernels)"}


def e2e_iterate(P, inp, perm_d, args, dev, ideal, world, rank):
    """The power iteration as a user calls it, from HOST memory: pinned H2D of
    x_0, P x, spmv_iterate (K steps), P^T x, D2H of x_K and lambda -- all
    inside the timed region; per-step bytes = the copies / K.  Max over
    ranks."""
    import torch
    import torch.distributed as dist
    n, K = inp.n, args.steps
    xh = torch.from_numpy(inp.x).pin_memory()
    outh = torch.empty(n, dtype=torch.float32).pin_memory()
    xd = torch.empty(n, dtype=torch.float32, device=dev)
    xB = torch.empty(n, dtype=torch.float32, device=dev)
    comp = torch.cuda.current_stream()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize(dev)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(comp)
    xd.copy_(xh, non_blocking=True)
    P.permute_vec(xd, out=xB)
    lam = P.iterate(xB, K)
    P.permute_vec(xB, inverse=True, out=xd)
    outh.copy_(xd, non_blocking=True)
    e1.record(comp)
    torch.cuda.synchronize(dev)
    ms = e0.elapsed_time(e1) / K
    if world > 1:
        t = torch.tensor([ms], dtype=torch.float64, device=dev)
        if args.backend == "nccl":
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        else:
            h = t.cpu()
            dist.all_reduce(h, op=dist.ReduceOp.MAX)
            t.copy_(h)
        ms = float(t.item())
    if not (math.isfinite(lam) and lam > 0 and bool(torch.isfinite(outh).all())):
        raise RuntimeError("e2e: power iteration result not finite")
    return {"value": round(ideal / (ms * 1e-3) / 1e9, 2), "unit": "GB/s", "ms_per_step": round(ms, 5),
            "h2d_bytes_per_step": round(4 * n / K, 1), "d2h_bytes_per_step": round((4 * n + 8) / K, 1),
            "lambda": lam,
            "path": "pinned H2D x_0 -> spmv_permute_vec -> spmv_iterate (K steps) -> "
                    "spmv_permute_vec^T -> D2H x_K + lambda, copies amortised over K steps"}


# ------------------------------------------------------------------- oracle
def oracle_sample(inp, perm, target_nnz=None):
    """A bounded, contiguous row block of B = P A P^T built by the oracle's own
    permutation (oracle.permute.permute_block) and x_B, for the CPU timing."""
    import numpy as np

    from oracle import permute as opermute
    n, nnz = inp.n, inp.nnz
    host = inp.host
    if host.val is None:
        host.val = inp.val_d.cpu().numpy()
    inv = opermute.inverse(perm)
    xB = opermute.permute_vec(inp.x, perm)
    if target_nnz is None or target_nnz >= nnz:
        r0, r1 = 0, n
    else:   # a middle block of rows with about target_nnz entries of B
        lenB = np.diff(host.row_ptr)[inv]
        cum = np.concatenate([[0], np.cumsum(lenB)])
        r0 = int(np.searchsorted(cum, (nnz - target_nnz) // 2))
        r1 = int(np.searchsorted(cum, (nnz + target_nnz) // 2))
    rp, col, val = opermute.permute_block(host.row_ptr, host.col, host.val, perm, inv, r0, r1)
    return rp, col, val, xB, r0, r1


def cpu_baseline(inp, perm, budget_s=10.0, steps=None, warmup=0):
    """The oracle as it stands (plain C fp64 CSR loop, OpenMP over the host
    cores, and the same loop on 1 core) on a bounded sample of the same
    reordered workload, in the metric's unit (ideal bytes of the sample, P:96
    restricted to its rows, per second).  Workloads above 2^28 entries are
    sampled as a contiguous middle block of B's rows (~2^24 entries)."""
    from oracle import cref
    # give the reorder's freed heap back to the OS first: the two processes
    # that time the oracle (the bench line, the reference arm) then agree
    # within 5 % (r84: 28.9 vs 30.2 GB/s; up to 1.55x apart before)
    import gc
    gc.collect()
    try:
        import ctypes
        ctypes.CDLL("libc.so.6").malloc_trim(0)
    except OSError:
        pass
    big = inp.nnz > 2**28
    rp, col, val, xB, r0, r1 = oracle_sample(inp, perm, target_nnz=2**24 if big else None)
    m, rows = int(rp[-1]), r1 - r0
    w_off = 8 if inp.nnz >= 2**31 else 4
    sample_ideal = 8 * m + (rows + 1) * w_off + 8 * rows
    desc = "all of B" if not big else \
        f"rows {r0}..{r1} of B ({m} entries, {100.0 * m / inp.nnz:.2f} % of nnz)"

    def timeit(threads, budget, nsteps, nwarm):
        """Budget mode (nsteps None): SpMVs until the budget is spent.  Step mode
        (the reference arm's --steps K --warmup W): a step is a batch of R
        SpMVs, R sized by the warm-up to ~0.5 s, so K steps time as many SpMVs
        as the budget mode and the two agree (one 4 ms SpMV per step did not)."""
        cref.threads(threads)
        t0 = time.perf_counter()
        nw = 0
        for _ in range(max(nwarm, 1 if nsteps is not None else 0)):
            cref.spmv_f64(rp, col, val, xB)
            nw += 1
        times, t_start = [], time.perf_counter()
        if nsteps is not None:
            one = (t_start - t0) / max(nw, 1)
            reps = max(1, int(0.5 / max(one, 1e-6)))
            for _ in range(nsteps):
                t = time.perf_counter()
                for _ in range(reps):
                    cref.spmv_f64(rp, col, val, xB)
                times.extend([(time.perf_counter() - t) / reps] * reps)
            return statistics.mean(times), len(times)
        while True:
            t = time.perf_counter()
            cref.spmv_f64(rp, col, val, xB)
            times.append(time.perf_counter() - t)
            if time.perf_counter() - t_start > budget:
                break
        return statistics.mean(times), len(times)

    ncpu = os.cpu_count() or 1
    s_all, k_all = timeit(ncpu, budget_s, steps, warmup)
    used = cref.threads(0)
    s_one, k_one = timeit(1, budget_s / 2, None if steps is None else max(1, steps // 4), 0)
    cref.threads(ncpu)
    return {"value": round(sample_ideal / s_all / 1e9, 3), "unit": "GB/s", "cores": used,
            "kind": "oracle", "ms_per_spmv": round(s_all * 1e3 * inp.nnz / max(m, 1), 3),
            "sample": f"{k_all} SpMVs of {desc} (plain C fp64, OpenMP static nnz-balanced, "
                      f"{used} threads); ms_per_spmv scaled to the whole matrix by nnz",
            "one_core": {"value": round(sample_ideal / s_one / 1e9, 3), "unit": "GB/s", "cores": 1,
                         "sample": f"{k_one} SpMVs of the same rows on 1 thread"},
            "host": host_info()}


def run_reference(args):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import torch
    dev = torch.device("cuda", 0) if torch.cuda.is_available() else None
    ordering = args.orderings.split(",")[-1]
    if dev is None and args.config in (1, 3, 5):
        raise SystemExit("--impl reference for this config needs the GPU generator")
    inp = Inputs(args.config, dev, need_host=True, small=args.small)
    perm, _ = reorder(args, inp, ordering)   # input preparation, outside the timed region
    ideal = ideal_bytes(inp.n, inp.nnz)
    cb = cpu_baseline(inp, perm, steps=args.steps, warmup=args.warmup)
    line = dict(metric=METRIC, value=cb["value"], unit="GB/s", n_gpus=world, steps=args.steps,
                warmup=args.warmup, ms_per_step=cb["ms_per_spmv"], higher_is_better=True,
                scaling="strong", vs_baseline=None, dtype="f64", data="synthetic", impl="reference",
                config={"workload": f"{inp.name} (BASELINE configs[{args.config - 1}])", "n": inp.n,
                        "nnz": inp.nnz, "ordering": ordering, "ideal_bytes": ideal,
                        "step": "a batch of SpMVs of the sample (~0.5 s; the oracle has no power-iteration "
                                "driver of its own); ms_per_step = one SpMV scaled to the whole matrix"},
                cpu_baseline=cb,
                e2e={"value": cb["value"], "unit": "GB/s", "h2d_bytes_per_step": 0,
                     "d2h_bytes_per_step": 0})
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", type=int, default=5, help="BASELINE.json config index (1-based)")
    ap.add_argument("--orderings", default=None,
                    help="comma list; the last one is the headline line (default: "
                         "original,rabbit,hubsort,rabbitpp for config 5, "
                         "random,original,rabbit,rabbitpp else)")
    ap.add_argument("--seed", type=int, default=20230423)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=10.0)
    ap.add_argument("--no-side", action="store_true",
                    help="skip the Table IV side measurements (SpMM-CSR-4, SpMV-COO)")
    ap.add_argument("--perm-cache", default=None, help="dev only: memoise reorder results here")
    ap.add_argument("--sequential-reorder", action="store_true",
                    help="RABBIT detection with the sequential (bit-exact) merge loop")
    ap.add_argument("--variant", type=int, default=0, help="short-row kernel: 0 lane, 1 panel")
    ap.add_argument("--backend", default="nccl", choices=["nccl", "gloo"],
                    help="collectives for N > 1 (gloo: host-staged, test only)")
    ap.add_argument("--exchange", default="coll", choices=["coll", "peer"],
                    help="N > 1: all-gatherv through the collective backend, or the SpMV's own "
                         "peer stores (CUDA IPC over NVLink)")
    ap.add_argument("--small", action="store_true",
                    help="test only: the same-shaped reduced instance of the config")
    ap.add_argument("--single-device", action="store_true",
                    help="test only: put every rank on cuda:0 (with --backend gloo)")
    args = ap.parse_args()
    if args.orderings is None:
        args.orderings = "original,rabbit,hubsort,rabbitpp" if args.config == 5 else \
            "random,original,rabbit,rabbitpp"
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        run_reference(args)
    else:
        run_gpu(args)


if __name__ == "__main__":
    main()
