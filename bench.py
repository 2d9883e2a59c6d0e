"""Benchmark of the community-reordered CSR SpMV hot path (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl reference]
                    [--config 2] [--orderings original,rabbit,rabbitpp]

N = 1: workload = BASELINE.json configs[1] (planted-community SBM, 4M rows,
64M nnz).  Input prep (host RABBIT / RABBIT++ reorder, GPU plan + P A P^T)
happens once and is reported separately (PAPER.md:221 amortisation).  A
step is one spmv_exec y_B = B x_B over the whole matrix with x_B, B resident
in HBM; L2 is flushed (512 MiB read) before every step, outside the CUDA
events that time it, so each step pays compulsory traffic like the paper's
ideal model.  value = ideal bytes / step time (GB/s);
runtime / ideal = peak / value.

N > 1 (torchrun): row-block power iteration on the same matrix, one rank per
GPU: step = exec_scaled + NCCL all-reduce (8 B) + in-place all-gather of x;
value = whole-job SpMV throughput (ideal bytes of the full B per step / max
over ranks of the step time); scaling "strong".

--impl reference: the oracle (plain C fp64 CSR loop, oracle/c) timed on the
host cores on the same workload, each step one full SpMV.
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


def load_workload(k: int):
    import synth
    t = time.perf_counter()
    w = synth.config(k)
    return w, time.perf_counter() - t


def ncu_traffic(workload: str, ordering: str):
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    if not os.path.exists(p):
        return None
    d = json.load(open(p))
    e = d.get(f"{workload}/{ordering}")
    return e if isinstance(e, dict) else None


def reorder_cached(args, name, A, ordering, planted=None):
    """spmv_reorder (host), optionally memoised on disk for development runs
    (--perm-cache DIR); the default bench run always recomputes.  "planted" is
    the generator's ground-truth order (SBM communities / stencil grid), a
    reference point, not a method of the paper."""
    import numpy as np
    from paper_conf_ispass_balajicjk23_b200 import spmv
    if ordering == "planted":
        if planted is None:
            raise SystemExit(f"workload {name} has no planted order")
        return planted.astype(np.int32), spmv.ReorderStats(
            **{f: 0 for f in spmv.ReorderStats.__dataclass_fields__})
    if args.perm_cache:
        f = os.path.join(args.perm_cache, f"{name}_{ordering}_{args.seed}.npz")
        if os.path.exists(f):
            d = np.load(f, allow_pickle=True)
            return d["perm"], spmv.ReorderStats(**d["stats"].item())
    perm, st = spmv.reorder(A.row_ptr, A.col, ordering, seed=args.seed)
    if args.perm_cache:
        os.makedirs(args.perm_cache, exist_ok=True)
        np.savez(f, perm=perm, stats=np.array(st.__dict__, dtype=object))
    return perm, st


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
    w, gen_s = load_workload(args.config)
    A = w.A
    hbm, peak_src = peaks()
    orderings = args.orderings.split(",")
    main = orderings[-1]
    results = {}
    rp_d = torch.from_numpy(A.row_ptr).to(dev)
    col_d = torch.from_numpy(A.col).to(dev)
    val_d = torch.from_numpy(A.val).to(dev)
    if A.nnz < 2**31:
        rp_d = rp_d.to(torch.int32)
    # L2 flush by READING 512 MiB (4x L2): leaves L2 full of clean lines, so the
    # timed step pays compulsory DRAM reads without write-backs of the flush
    flush = torch.zeros(512 * 2**20 // 4, dtype=torch.float32, device=dev)
    sink = torch.zeros((), dtype=torch.float32, device=dev)

    def flush_l2():
        torch.sum(flush, dim=0, out=sink)

    # a dedicated (non-legacy) stream: the L2 access-policy window of spmv_exec
    # is a stream attribute and cannot be set on the legacy default stream
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    line = None
    for ordering in orderings:
        perm, st = reorder_cached(args, w.name, A, ordering, w.planted)
        if ordering == main:
            main_perm = perm
        perm_d = torch.from_numpy(perm).to(dev)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        P = spmv.Plan(rp_d, col_d, val_d, perm_d, world=world, rank=rank, variant=args.variant)
        torch.cuda.synchronize()
        plan_s = time.perf_counter() - t0
        info = P.info()
        x_d = torch.from_numpy(w.x).to(dev)
        xB = P.permute_vec(x_d)
        if world > 1:
            xB = P.pad_vec(xB, to_padded=True)
        ideal = 2 * A.n * 4 + (A.n + 1) * info["offset_bytes"] + 2 * A.nnz * 4
        ideal_p96 = 2 * A.n * 4 + (A.n + 1 + 2 * A.nnz) * 4
        launches = info["exec_launches"]
        is_main = ordering == main
        fx = None
        K = args.steps if is_main else max(10, args.steps // 4)
        if world == 1:
            y = torch.empty(A.n, dtype=torch.float32, device=dev)

            def step():
                P.exec(xB, y)
        else:
            loc = pdist.PlanLocal(P)
            xa, xb = xB, torch.empty_like(xB)
            ss = torch.zeros(2, dtype=torch.float64, device=dev)
            state = {"t": 0, "xa": xa, "xb": xb, "ss_in": None}
            M, off, nr = loc.x_stride, loc.y_offset, loc.nrows

            if args.exchange == "fused":  # y rows stored into every peer's x
                fx = pdist.FusedExchange(P, dev, host_staged=args.backend != "nccl")
                fx.x.copy_(xB)

            def step():
                t = state["t"]
                ss_out = ss[t & 1:(t & 1) + 1]
                if fx is not None:
                    fx.step(state["ss_in"], ss_out)
                    state["ss_in"] = ss_out
                    state["t"] = t + 1
                    return
                P.exec_scaled(state["xa"], state["xb"][off:off + nr], state["ss_in"], ss_out)
                if args.backend == "nccl":
                    dist.all_reduce(ss_out)
                    dist.all_gather_into_tensor(state["xb"], state["xb"][off:off + M])
                else:  # gloo test path: host staging
                    h = ss_out.cpu()
                    dist.all_reduce(h)
                    ss_out.copy_(h)
                    hx = state["xb"].cpu()
                    dist.all_gather_into_tensor(hx, hx[off:off + M].clone())
                    state["xb"].copy_(hx)
                state["ss_in"] = ss_out
                state["xa"], state["xb"] = state["xb"], state["xa"]
                state["t"] = t + 1
            launches += 1  # exec_scaled's fixed-order norm reduction
        for _ in range(args.warmup):
            flush_l2()
            step()
        torch.cuda.synchronize()
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
              for _ in range(K)]
        clocks = Clocks(local) if is_main and rank == 0 else None
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        if clocks:
            clocks.start()
            time.sleep(0.3)
        wall0 = time.perf_counter()
        for i in range(K):
            flush_l2()
            ev[i][0].record(stream)
            step()
            ev[i][1].record(stream)
        torch.cuda.synchronize()
        wall = time.perf_counter() - wall0
        if world > 1:
            dist.barrier()
        ck = clocks.stop() if clocks else None
        times = [a.elapsed_time(b) for a, b in ev]
        ms = sum(times) / K
        if world > 1:
            t = torch.tensor([ms], dtype=torch.float64, device=dev)
            if args.backend == "nccl":
                dist.all_reduce(t, op=dist.ReduceOp.MAX)
            else:
                h = t.cpu()
                dist.all_reduce(h, op=dist.ReduceOp.MAX)
                t.copy_(h)
            ms = float(t.item())
        # warm (no flush) back-to-back
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(K):
            step()
        e1.record(stream)
        torch.cuda.synchronize()
        warm_ms = e0.elapsed_time(e1) / K
        graph_ms = None
        if world == 1 and ideal < 256 * 2**20:
            # small (L2-resident) matrices: launch overhead dominates a single
            # exec, so also time G execs captured in one CUDA graph (warm)
            G = 200
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=stream):
                for _ in range(G):
                    step()
            g.replay()
            torch.cuda.synchronize()
            e0.record(stream)
            for _ in range(5):
                g.replay()
            e1.record(stream)
            torch.cuda.synchronize()
            graph_ms = e0.elapsed_time(e1) / (5 * G)
        gbs = ideal / (ms * 1e-3) / 1e9
        res = {"ms": ms, "ms_median": statistics.median(times), "warm_ms": warm_ms,
               "graph_warm_ms": graph_ms,
               "gbs_ideal_over_t": gbs, "gflops": 2 * A.nnz / (ms * 1e-3) / 1e9,
               "runtime_over_ideal": hbm / gbs, "reorder_s": st.seconds, "plan_permute_s": plan_s,
               "insularity": st.insularity, "insular_frac": st.insular_frac,
               "n_communities": st.n_communities, "largest_comm_frac": st.largest_comm_frac,
               "modularity": st.modularity, "skew": st.skew, "hubs": st.n_hubs,
               "H": info["hot_prefix"], "tiles": info["n_tiles"], "cta_rows": info["n_cta_rows"],
               "hub_rows": info["n_hub_rows"], "l2_window_bytes": P.info()["l2_window_bytes"],
               "stream_evict_first": info["stream_evict_first"]}
        if world == 1 and not args.no_side:
            # the paper's Table IV kernels on the same reordered matrix
            res["spmm4"] = side_measure("spmm4", P, A, info, K, flush_l2, stream, dev, hbm)
            res["coo"] = side_measure("coo", P, A, info, K, flush_l2, stream, dev, hbm)
        tr = ncu_traffic(w.name, ordering)
        if tr:
            res["dram_over_ideal_ncu"] = tr.get("dram_bytes", 0) / ideal
        results[ordering] = res
        if is_main:
            if world == 1:
                e2e = e2e_measure(P, A, w.x, args, dev, ideal)
            else:
                state["xcur"] = (lambda: fx.x) if fx is not None else (lambda: state["xa"])
                e2e = e2e_dist_measure(P, loc, w.x, perm, step_state=state, step=step, args=args,
                                       dev=dev, ideal=ideal, world=world)
            line = dict(metric=METRIC, value=round(gbs, 2), unit="GB/s", n_gpus=world, steps=K,
                        warmup=args.warmup, ms_per_step=round(ms, 5), higher_is_better=True,
                        scaling="strong", vs_baseline=None, dtype="f32",
                        data="synthetic")
            line["config"] = {"workload": f"{w.name} (BASELINE configs[{args.config - 1}])",
                              "n": A.n, "nnz": A.nnz, "ordering": ordering,
                              "parallelism": f"row-block x{world}" if world > 1 else "1 GPU",
                              "step": "spmv_exec" if world == 1 else
                              ("exec_scaled_bcast (fused NVLink peer stores) + all_reduce (power iteration)"
                                       if args.exchange == "fused" else
                                       "exec_scaled + all_reduce + all_gather (power iteration)"),
                              "l2": "flushed before every step (512 MiB read, outside the events)",
                              "ideal_bytes": ideal, "ideal_bytes_paper_4B_offsets": ideal_p96,
                              "kernel_variant": ["lane", "panel"][args.variant],
                              "wall_s_timed_region": round(wall, 4)}
            line["runtime_over_ideal"] = round(hbm / gbs, 4)
            line["gflops"] = round(2 * A.nnz / (ms * 1e-3) / 1e9, 2)
            kern_bytes = ideal
            line["roofline"] = {"bound": "hbm", "achieved": round(kern_bytes / (ms * 1e-3) / 1e9, 2),
                                "peak": hbm, "unit": "GB/s",
                                "frac": round(kern_bytes / (ms * 1e-3) / 1e9 / hbm, 4),
                                "traffic": tr.get("dram_bytes") if tr else None,
                                "kernel": ["k_lane", "k_panel"][args.variant] + " (+k_cta_rows/k_hub_* if present)",
                                "peak_source": peak_src,
                                "algorithmic_bytes_per_launch": kern_bytes}
            line["e2e"] = e2e
            line["gpu_launches"] = launches * K
            line["clocks"] = ck
            line["input_prep"] = {"generate_s": round(gen_s, 3), "reorder_s": round(st.seconds, 3),
                                  "plan_permute_s": round(plan_s, 4)}
        if fx is not None:
            fx.close()
        P.close()
    line["orderings"] = {k: {kk: (round(vv, 5) if isinstance(vv, float) else vv)
                             for kk, vv in v.items()} for k, v in results.items()}
    if "random" in results or "original" in results:
        base = results.get("original") or results.get("random")
        if base and main in results:
            saving = base["ms"] - results[main]["ms"]
            line["amortization_iters_vs_" + ("original" if "original" in results else "random")] = \
                (results[main]["reorder_s"] * 1e3 / saving) if saving > 0 else None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        from oracle import permute as opermute
        B = opermute.permute_csr_scipy(A.n, A.row_ptr, A.col, A.val, main_perm)
        Bm = type("M", (), {"row_ptr": B[0], "col": B[1], "val": B[2]})()
        line["cpu_baseline"] = cpu_baseline(Bm, opermute.permute_vec(w.x, main_perm),
                                            ideal_bytes=line["config"]["ideal_bytes"])
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def side_measure(kind, P, A, info, K, flush_l2, stream, dev, hbm):
    """Table IV kernels on the same plan, cold L2 like the
    SpMV steps, ideal traffic "updated according to the kernel":
      spmm4: 8 NZ + (N+1) w_off + 16 N (X) + 16 N (Y)
      coo:   12 NZ + 4 N (x) + 4 N (y)"""
    import torch
    if kind == "spmm4":
        X = torch.empty((A.n, 4), dtype=torch.float32, device=dev).uniform_(-1, 1)
        Y = torch.empty_like(X)
        ideal = 32 * A.n + (A.n + 1) * info["offset_bytes"] + 8 * A.nnz
        flops = 8 * A.nnz

        def run():
            P.exec_spmm4(X, Y)
    else:
        X = torch.empty(A.n, dtype=torch.float32, device=dev).uniform_(-1, 1)
        Y = torch.empty_like(X)
        ideal = 8 * A.n + 12 * A.nnz
        flops = 2 * A.nnz

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


def e2e_measure(P, A, x_host, args, dev, ideal):
    """Same metric through the public API with HOST buffers: pinned H2D of x,
    P x, exec, P^T y, D2H of y -- all inside the timed region.  Steps are
    software-pipelined over two buffer slots on three streams (H2D copy engine,
    compute, D2H copy engine), as a serving loop would run it: step i+1's
    upload and step i-1's download overlap step i's kernels."""
    import torch
    comp = torch.cuda.current_stream()
    s_in, s_out = torch.cuda.Stream(), torch.cuda.Stream()
    xh = torch.from_numpy(x_host).pin_memory()
    yh = [torch.empty(A.n, dtype=torch.float32).pin_memory() for _ in range(2)]
    xd = [torch.empty(A.n, dtype=torch.float32, device=dev) for _ in range(2)]
    yd = [torch.empty(A.n, dtype=torch.float32, device=dev) for _ in range(2)]
    xB = torch.empty(A.n, dtype=torch.float32, device=dev)
    yB = torch.empty_like(xB)
    ev = {k: [torch.cuda.Event() for _ in range(2)] for k in ("h2d", "comp", "d2h")}
    started = [False, False]

    def step(i):
        b = i & 1
        if started[b]:
            s_in.wait_event(ev["comp"][b])     # xd[b] no longer read
        with torch.cuda.stream(s_in):
            xd[b].copy_(xh, non_blocking=True)
        ev["h2d"][b].record(s_in)
        comp.wait_event(ev["h2d"][b])
        if started[b]:
            comp.wait_event(ev["d2h"][b])      # yd[b] already downloaded
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
    # the downloaded y of the last step is the full public-API result
    xd[0].copy_(xh)
    P.permute_vec(xd[0], out=xB)
    P.exec(xB, yB)
    P.permute_vec(yB, inverse=True, out=yd[0])
    if not torch.equal(yd[0].cpu(), yh[(K - 1) & 1]):
        raise RuntimeError("e2e: pipelined result differs from a direct call")
    return {"value": round(ideal / (ms * 1e-3) / 1e9, 2), "unit": "GB/s", "ms_per_step": round(ms, 5),
            "h2d_bytes_per_step": 4 * A.n, "d2h_bytes_per_step": 4 * A.n,
            "path": "pinned H2D x -> spmv_permute_vec -> spmv_exec -> spmv_permute_vec^T -> D2H y "
                    "(two slots, copy engines overlapped with the kernels)"}


def e2e_dist_measure(P, loc, x_host, perm, step_state, step, args, dev, ideal, world):
    """N > 1: per step, pinned H2D of this rank's slice of x_B into its segment of
    the padded x, the distributed step (exec_scaled + all-reduce + all-gather),
    D2H of the 8-byte norm; max over ranks of the per-step time."""
    import torch
    import torch.distributed as dist
    b0, b1 = P.export_partition()[loc.rank], P.export_partition()[loc.rank + 1]
    xB = P.permute_vec(torch.from_numpy(x_host).to(dev))  # setup, outside the timed region
    xs = xB[b0:b1].cpu().pin_memory()
    ssh = torch.empty(1, dtype=torch.float64).pin_memory()
    off = loc.y_offset

    def e2e_step():
        step_state["xcur"]()[off:off + (b1 - b0)].copy_(xs, non_blocking=True)
        step()
        ssh.copy_(step_state["ss_in"], non_blocking=True)

    for _ in range(args.warmup):
        e2e_step()
    torch.cuda.synchronize()
    dist.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(args.steps):
        e2e_step()
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / args.steps
    t = torch.tensor([ms], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX) if args.backend == "gloo" else None
    if args.backend == "nccl":
        td = t.to(dev)
        dist.all_reduce(td, op=dist.ReduceOp.MAX)
        t = td.cpu()
    ms = float(t.item())
    return {"value": round(ideal / (ms * 1e-3) / 1e9, 2), "unit": "GB/s", "ms_per_step": round(ms, 5),
            "h2d_bytes_per_step": 4 * int(P.info()["n"]), "d2h_bytes_per_step": 8 * world,
            "path": "pinned H2D of each rank's x slice -> spmv_exec_scaled -> NCCL all-reduce "
                    "+ all-gather -> D2H of the norm (summed over ranks)"}


# ------------------------------------------------------------------- oracle
def cpu_baseline(A, x, ideal_bytes, budget_s=10.0, steps=None, warmup=0):
    """The oracle as it stands (plain C fp64 CSR loop, OpenMP over all host
    cores) on the same workload; bounded sample of full SpMVs."""
    from oracle import cref
    threads = cref.threads()
    for _ in range(warmup):
        cref.spmv_f64(A.row_ptr, A.col, A.val, x)
    times = []
    t_start = time.perf_counter()
    while True:
        t = time.perf_counter()
        cref.spmv_f64(A.row_ptr, A.col, A.val, x)
        times.append(time.perf_counter() - t)
        if steps is not None:
            if len(times) >= steps:
                break
        elif time.perf_counter() - t_start > budget_s:
            break
    s = statistics.mean(times)
    return {"value": round(ideal_bytes / s / 1e9, 3), "unit": "GB/s", "cores": threads,
            "kind": "oracle", "ms_per_spmv": round(s * 1e3, 3),
            "sample": f"{len(times)} full SpMVs of the workload (plain C fp64, OpenMP static nnz-balanced)"}


def run_reference(args):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    w, _ = load_workload(args.config)
    A = w.A
    from paper_conf_ispass_balajicjk23_b200 import spmv
    perm, _ = spmv.reorder(A.row_ptr, A.col, args.orderings.split(",")[-1], seed=args.seed)
    from oracle import permute
    Bp, Bc, Bv = permute.permute_csr_scipy(A.n, A.row_ptr, A.col, A.val, perm.astype("int64"))
    xB = permute.permute_vec(w.x, perm)
    ideal = 2 * A.n * 4 + (A.n + 1) * (8 if A.nnz >= 2**31 else 4) + 2 * A.nnz * 4
    cb = cpu_baseline(type("M", (), {"row_ptr": Bp, "col": Bc, "val": Bv})(), xB, ideal,
                      steps=args.steps, warmup=args.warmup)
    ms = cb["ms_per_spmv"]
    line = dict(metric=METRIC, value=cb["value"], unit="GB/s", n_gpus=world, steps=args.steps,
                warmup=args.warmup, ms_per_step=ms, higher_is_better=True, scaling="strong",
                vs_baseline=None, dtype="f64", data="synthetic", impl="reference",
                config={"workload": f"{w.name} (BASELINE configs[{args.config - 1}])", "n": A.n,
                        "nnz": A.nnz, "ordering": args.orderings.split(",")[-1],
                        "ideal_bytes": ideal},
                cpu_baseline=cb,
                e2e={"value": cb["value"], "unit": "GB/s", "h2d_bytes_per_step": 0,
                     "d2h_bytes_per_step": 0})
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", type=int, default=2, help="BASELINE.json config index (1-based)")
    ap.add_argument("--orderings", default="original,rabbit,rabbitpp",
                    help="comma list; the last one is the headline line")
    ap.add_argument("--seed", type=int, default=20230423)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-side", action="store_true",
                    help="skip the Table IV side measurements (SpMM-CSR-4, SpMV-COO)")
    ap.add_argument("--perm-cache", default=None, help="dev only: memoise reorder results here")
    ap.add_argument("--variant", type=int, default=0, help="short-row kernel: 0 lane, 1 panel")
    ap.add_argument("--backend", default="nccl", choices=["nccl", "gloo"],
                    help="collectives for N > 1 (gloo: host-staged, test only)")
    ap.add_argument("--exchange", default="nccl", choices=["nccl", "fused"],
                    help="N > 1: NCCL all-gather of x, or the fused exec + NVLink peer stores")
    ap.add_argument("--single-device", action="store_true",
                    help="test only: put every rank on cuda:0 (with --backend gloo)")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        run_reference(args)
    else:
        run_gpu(args)


if __name__ == "__main__":
    main()
