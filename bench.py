#!/usr/bin/env python
"""bench.py — FP64 GFLOP/s (n^3/3) of the Enhanced Online-ABFT Cholesky on B200, ABFT overhead %.

Default workload (BASELINE.json configs[3] at N=1, the north_star's headline point):
n = 32768, nb = 512, random SPD (reading A15 generator, seed = n), fault-free, ABFT on.
A "step" is one complete abft_potrf (encode, V1-V6, POTRF, TRSM, trailing update) over a fresh
copy of the matrix, resident in HBM (8 GiB > 126 MB L2, so no L2 flush is needed).

Timing: W warm-up steps, then exactly K steps, each bracketed by CUDA events on the launching
stream (the restore of the input between steps is outside the events); barrier + synchronize
before and after the timed loop; max over ranks. nvidia-smi samples clocks during the timed loop.

Extra measurements reported on the same line (same workload, not part of `value`):
  abft_off       the same kernels with every checksum operation removed (overhead %)
  injected       C3-style computing + storage errors, one of each per iteration
  e2e            abft_potrf_host on pinned host memory: H2D + factorisation + D2H per step
  roofline       dominant kernel (trailing DMMA update) from the library's per-phase CUDA events
  cpu_baseline   the CPU oracle on a bounded sample (rank 0, N=1)
  cusolver       torch.linalg.cholesky (cuSOLVER dpotrf, vendor context, no ABFT)

--impl reference: the oracle (the only reference implementation this paper-only tier has), timed
on the host cores on a bounded sample of the same workload per step.
"""
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

FP64_DMMA_PEAK_TFLOPS = 37.1   # measured: tools/fp64_peak.cu, register-resident DMMA (profiles/fp64_peak_r01.txt)
HBM_PEAK_FALLBACK = 6555.8


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--n", type=int, default=32768)
    ap.add_argument("--nb", type=int, default=512)
    ap.add_argument("--no-extras", action="store_true", help="main metric only (for ncu launch lists)")
    ap.add_argument("--oracle-n", type=int, default=6144, help="cpu_baseline sample size")
    return ap.parse_args()


def measured_peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


# ---- clocks sampler ----------------------------------------------------------------------
class Clocks:
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index=0):
        self.index, self.lines, self.proc = index, [], None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [x.strip() for x in ln.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                mx = float(parts[1])
            except ValueError:
                continue
            for nm, v in zip(names, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


def update_traffic(n, nb):
    """Measured DRAM bytes per update launch (ncu, committed under profiles/) for this workload."""
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "update_traffic_r01.json")))
        if f"run_once.py {n} {nb}" in d.get("command", ""):
            return round(d["traffic_bytes_per_launch"])
    except Exception:
        pass
    return None


# ---- the oracle as CPU baseline / reference arm ---------------------------------------------
def oracle_sample(n_s, nb):
    import numpy as np
    import oracle
    import synthetic as syn
    A = syn.spd_matrix(n_s)
    t0 = time.perf_counter()
    r = oracle.potrf(A, nb)
    dt = time.perf_counter() - t0
    assert r.status == 0
    return n_s ** 3 / 3 / dt / 1e9, dt, oracle.num_threads()


def run_reference(args, rank, world):
    if rank != 0:
        return
    n_s = min(args.n, 4096)
    vals = []
    for i in range(args.warmup + args.steps):
        g, dt, cores = oracle_sample(n_s, args.nb)
        if i >= args.warmup:
            vals.append((g, dt))
    value = statistics.median(v[0] for v in vals)
    sample = f"oracle potrf n={n_s} nb={args.nb} per step (bounded sample of the n={args.n} workload), fault-free, ABFT on"
    line = {"impl": "reference", "metric": "FP64 GFLOP/s (n^3/3) with online ABFT", "value": round(value, 3),
            "unit": "GFLOP/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(1e3 * statistics.median(v[1] for v in vals), 3), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"C4: n={args.n} nb={args.nb} random SPD (A15), fault-free", "n": args.n,
                       "nb": args.nb},
            "cpu_baseline": {"value": round(value, 3), "unit": "GFLOP/s", "cores": cores, "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": round(value, 3), "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---- our arm -------------------------------------------------------------------------------
def main():
    args = parse()
    rank = int(os.environ.get("RANK", 0))
    world = int(os.environ.get("WORLD_SIZE", 1))
    if args.impl == "reference":
        return run_reference(args, rank, world)

    import numpy as np
    import torch
    import paper_conf_ipps_chenlc16_b200 as P

    local = int(os.environ.get("LOCAL_RANK", 0))
    torch.cuda.set_device(local)
    dist = world > 1
    if dist:
        import torch.distributed as tdist
        tdist.init_process_group("nccl", device_id=torch.device("cuda", local))
    n, nb = args.n, args.nb
    flops = n ** 3 / 3
    stream = torch.cuda.current_stream()
    # input: generated on the device by the A15 generator, kept pristine for restores
    A0 = torch.empty(n, n, dtype=torch.float64, device="cuda").T
    assert P.abft_gen_spd(n, A0) == 0
    comm = None
    if dist:
        # 1D block-cyclic: this rank keeps its block columns (J mod world == rank)
        idx = torch.cat([torch.arange(J * nb, (J + 1) * nb) for J in P.owned_blocks(n // nb, rank, world)])
        A0 = A0.T[idx.cuda()].contiguous().T          # column-major n x n_local
        torch.cuda.synchronize()
        nid = P.nccl_id_exchange()
        st, comm = P.abft_comm_init(world, nid, rank)
        assert st == 0, "abft_comm_init failed"
    A = torch.empty_like(A0.T).T

    def factor(opt, inj=None, cap=4096):
        if dist:
            return P.abft_potrf_dist(n, nb, A, comm, rank, world, inj=inj, opt=opt, report=True, cap=cap)
        return P.abft_potrf_ex(n, nb, A, inj=inj, opt=opt, report=True, cap=cap)

    def barrier():
        if dist:
            import torch.distributed as tdist
            tdist.barrier()
        torch.cuda.synchronize()

    def run_steps(opt, inj=None, steps=args.steps, warmup=args.warmup, check=True):
        times, reps = [], []
        for i in range(warmup + steps):
            A.copy_(A0)
            if i == warmup:
                barrier()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            st, rep = factor(opt, inj)
            e1.record(stream)
            e1.synchronize()
            if check:
                assert st == 0, f"abft_potrf status {st}"
            if i >= warmup:
                times.append(e0.elapsed_time(e1))
                reps.append(rep)
        barrier()
        return times, reps

    # ---- main metric: ABFT on, fault-free, per-phase profile on -------------------------
    with Clocks(local) as clk:
        times, reps = run_steps(P.options(profile=True))
    prof = P.abft_last_profile()
    launches = P.abft_last_launch_count()
    ms_local = sum(times) / len(times)
    ms = ms_local
    if dist:
        import torch.distributed as tdist
        t = torch.tensor([ms_local], device="cuda")
        tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
        ms = t.item()
    # one n x n factorisation per step (strong scaling across ranks at N > 1)
    value = flops / (ms * 1e-3) / 1e9
    upd = prof.get("update", {})
    achieved = upd["flops"] / (upd["ms"] * 1e-3) / 1e12 if upd.get("ms") else None
    line = {
        "metric": "FP64 GFLOP/s (n^3/3) with online ABFT", "value": round(value, 2), "unit": "GFLOP/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 3),
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
        "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"C4: n={n} nb={nb} random SPD (A15 generator, seed=n), fault-free, Enhanced "
                               f"Online-ABFT on (K=1), 1 GPU per rank", "n": n, "nb": nb,
                   "l2": "inputs (8 GiB) larger than L2; restore copy between steps outside the CUDA events",
                   "parallelism": f"1D block-cyclic x{world}, NCCL panel broadcast" if world > 1 else "single GPU"},
        "gpu_launches": int(launches) * args.steps,
        "roofline": {"bound": "tensor", "kernel": "k_update_ws (warp-specialised DMMA, 128x64 tiles, 2 CTAs/SM) trailing SYRK update + checksum rows",
                     "achieved": round(achieved, 3) if achieved else None,
                     "peak": FP64_DMMA_PEAK_TFLOPS, "unit": "TFLOP/s",
                     "frac": round(achieved / FP64_DMMA_PEAK_TFLOPS, 4) if achieved else None,
                     "traffic": update_traffic(n, nb),
                     "traffic_source": "ncu dram__bytes_read.sum + dram__bytes_write.sum per k_update_ws launch, "
                                       "averaged over every launch of one factorisation of this workload "
                                       "(profiles/update_traffic_r01.json, cold-cache serialised replay)",
                     "peak_source": "measured FP64 DMMA register-resident loop on this pool's B200 "
                                    "(MEASURED_PEAKS.json has no FP64 entry)",
                     "share_of_step": round(upd["ms"] / ms_local, 4) if upd.get("ms") else None},
        "whole_path_frac_of_fp64_peak": round(value / world / 1e3 / FP64_DMMA_PEAK_TFLOPS, 4),
        "abft_events": int(reps[-1]["n_events"]),
        "phases_ms_per_step": {k: round(v["ms"], 3) for k, v in prof.items()},
        "library_device_ms": round(1e3 * sum(r["seconds"] for r in reps) / len(reps), 3),
    }
    line["clocks"] = clk.summary()
    # bandwidth-bound check kernels: algorithmic bytes / device time (events around each phase)
    hbm_peak = measured_peaks().get("hbm_gbs", HBM_PEAK_FALLBACK)
    hbm = {}
    for ph in ("encode", "v6", "v1v2", "v4", "v5", "writeback"):
        v = prof.get(ph)
        if v and v["ms"] > 0 and v["bytes"] > 0:
            gbs = v["bytes"] / (v["ms"] * 1e-3) / 1e9
            hbm[ph] = {"GB/s": round(gbs, 1), "frac": round(gbs / hbm_peak, 3)}
    line["hbm_kernels"] = {"peak_GBps": hbm_peak, "peak_source": "MEASURED_PEAKS.json hbm_gbs", **hbm,
                           "note": "v1v2/v4/writeback run on the look-ahead stream concurrently with the "
                                   "update GEMM, so their device time includes waiting for SM slots"}

    if not args.no_extras and world == 1:   # extras are single-GPU runs (no collectives)
        # ABFT off: the same kernels without checksum work
        t_off, _ = run_steps(P.options(abft_enabled=False), steps=max(1, args.steps), warmup=1)
        ms_off = sum(t_off) / len(t_off)
        line["abft_off"] = {"value": round(flops / (ms_off * 1e-3) / 1e9, 2), "ms_per_step": round(ms_off, 3)}
        line["abft_overhead_pct"] = round(100 * (ms_local - ms_off) / ms_off, 3)
        # injected: one storage + one computing error per iteration (C3-style)
        import synthetic as syn
        specs = [s for s in syn.mixed_injections(n, nb) if s["hook"] != "RECV"]
        inj = syn.inj_array(specs)
        t_inj, rep_inj = run_steps(P.options(), inj=inj, steps=max(1, args.steps), warmup=1, check=False)
        r0 = rep_inj[-1]
        line["injected"] = {"value": round(flops / (sum(t_inj) / len(t_inj) * 1e-3) / 1e9, 2),
                            "injections": len(specs), "events": int(r0["n_events"]),
                            "corrected": int(r0["n_data"] + r0["n_nonfinite"] + r0["n_chk1"] + r0["n_chk2"]),
                            "uncorrectable": int(r0["n_uncorrectable"])}
        # NEXT-1: the paper's own left-looking order (MAGMA Alg. 1) with Table I's verification, and
        # Opt. 3 (verify every K iterations), next to the right-looking default
        orders = {}
        for order in ("right", "left"):
            for abft_on, Kv in ((True, 1), (True, 3), (False, 1)):
                to, ro = run_steps(P.options(abft_enabled=abft_on, K=Kv, order=order), steps=1, warmup=1)
                orders[f"{order}_{'abft' if abft_on else 'off'}_K{Kv}"] = {
                    "ms": round(to[0], 2), "value": round(flops / (to[0] * 1e-3) / 1e9, 1),
                    "tile_checks": int(ro[0]["n_checks"])}
        line["orders"] = orders
        # Table VII/VIII analog on B200 (NEXT-2): the three schemes x {no error, computation error,
        # memory error between verification and access}; Online/Offline re-do the factorisation
        # when an error propagated
        B_ = nb
        faults = {"no_error": [], "computation_error": [dict(k=2, hook="UPDATE_OUT", row=n - 700, col=n // 2, bit=50)],
                  "memory_error": [dict(k=3, hook="REST", row=3 * B_ + 100, col=3 * B_ + 50, bit=50)]}
        table = {}
        for mode in ("enhanced", "online", "offline"):
            table[mode] = {}
            for fname, specs in faults.items():
                injf = syn.inj_array(specs) if specs else None
                tf, rf = run_steps(P.options(mode=mode), inj=injf, steps=1, warmup=1, check=True)
                table[mode][fname] = {"ms": round(tf[0], 2), "value": round(flops / (tf[0] * 1e-3) / 1e9, 1),
                                      "reruns": int(rf[0]["reruns"]), "events": int(rf[0]["n_events"])}
        # NEXT-4: two errors in one column of a block (beyond what two checksums locate):
        # Enhanced stops with UNCORRECTABLE; Enhanced + re-do re-runs once from the saved input
        dbl = syn.inj_array([dict(k=3, hook="REST", row=3 * B_ + 100, col=3 * B_ + 50, bit=50),
                             dict(k=3, hook="REST", row=3 * B_ + 140, col=3 * B_ + 50, bit=51)])
        table["two_errors_in_a_column"] = {}
        for mode in ("enhanced", "enhanced_redo"):
            tf, rf = run_steps(P.options(mode=mode), inj=dbl, steps=1, warmup=1, check=False)
            table["two_errors_in_a_column"][mode] = {
                "ms": round(tf[0], 2), "status": "uncorrectable" if rf[0]["n_uncorrectable"] and not rf[0]["reruns"]
                else "ok", "reruns": int(rf[0]["reruns"]), "events": int(rf[0]["n_events"])}
        table["paper_context_seconds"] = {
            "Tardis_M2075_n20480": {"enhanced": [10.6572, 10.6614, 10.6678], "online": [10.5067, 10.5244, 22.625],
                                    "offline": [10.4489, 21.3942, 21.2631], "src": "PAPER.md:366-368"},
            "Bulldozer64_K40c_n30720": {"enhanced": [8.84598, 8.92538, 8.914928], "online": [8.64649, 8.69622, 21.4162],
                                        "offline": [8.64265, 21.4472, 21.3511], "src": "PAPER.md:374-377"}}
        line["schemes_table"] = table
        # e2e through the host C-ABI entry (pinned host memory, H2D + D2H inside the timing)
        del A
        torch.cuda.empty_cache()
        h0 = torch.empty(n * n, dtype=torch.float64, pin_memory=True)
        h = torch.empty(n * n, dtype=torch.float64, pin_memory=True)
        h0.copy_(A0.T.contiguous().view(-1))     # row-major of A0^T == column-major of A0
        e2e_t = []
        for i in range(1 + max(1, args.steps)):
            h.copy_(h0)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            st, _ = P.abft_potrf_host(n, nb, h.data_ptr(), lda=n, report=True, cap=16)
            t1 = time.perf_counter()
            assert st == 0
            if i >= 1:
                e2e_t.append(t1 - t0)
        te = sum(e2e_t) / len(e2e_t)
        # H2D and D2H: each block column from its diagonal block down (rows k*nb..n-1); the D2H of a
        # finished block column of L runs while the factorisation continues
        nblk = n // nb
        d2h = 8 * nb * (nblk * n - nb * nblk * (nblk - 1) // 2)
        line["e2e"] = {"value": round(flops / te / 1e9, 2), "unit": "GFLOP/s", "h2d_bytes_per_step": d2h,
                       "d2h_bytes_per_step": d2h, "ms_per_step": round(te * 1e3, 3),
                       "note": "wall clock around abft_potrf_host on pinned host memory; H2D of each block column "
                               "from its diagonal block down (what uplo=L reads); L's block columns are copied back "
                               "as they are finished, overlapped with the trailing updates"}
        del h, h0
        # vendor context: cuSOLVER dpotrf via torch (no ABFT)
        try:
            X = A0.T.contiguous()
            torch.linalg.cholesky(X)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(); torch.linalg.cholesky(X); e1.record(); e1.synchronize()
            line["cusolver_dpotrf_context"] = {"value": round(flops / (e0.elapsed_time(e1) * 1e-3) / 1e9, 2),
                                               "note": "vendor library, no ABFT, context only"}
            del X
        except Exception as ex:  # pragma: no cover
            line["cusolver_dpotrf_context"] = {"error": str(ex)[:100]}
        # CPU oracle, bounded sample
        if world == 1:
            g, dt, cores = oracle_sample(args.oracle_n, nb)
            line["cpu_baseline"] = {"value": round(g, 3), "unit": "GFLOP/s", "cores": cores, "kind": "oracle",
                                    "sample": f"oracle potrf n={args.oracle_n} nb={nb} (same nb, "
                                              f"{(args.oracle_n / n) ** 3:.4f} of the workload's flops), "
                                              f"fault-free, ABFT on, {dt:.1f} s"}
        # the other BASELINE configurations, one GPU, fault-free, ABFT on (median of the steps)
        others = {}
        for (cn, cnb, cst) in ((4096, 256, 5), (16384, 512, 5), (98304, 1024, 1)):
            try:
                del A0, A
            except NameError:
                pass
            torch.cuda.empty_cache()
            Ac = torch.empty(cn, cn, dtype=torch.float64, device="cuda").T
            Ac0 = torch.empty_like(Ac.T).T
            P.abft_gen_spd(cn, Ac0)
            ts = []
            for i in range(1 + cst):
                Ac.copy_(Ac0)
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
                e0.record(stream)
                st, _ = P.abft_potrf_ex(cn, cnb, Ac, report=True, cap=16)
                e1.record(stream); e1.synchronize()
                assert st == 0
                if i >= 1:
                    ts.append(e0.elapsed_time(e1))
            tm = statistics.median(ts)
            others[f"n{cn}_nb{cnb}"] = {"value": round(cn ** 3 / 3 / (tm * 1e-3) / 1e9, 1), "unit": "GFLOP/s",
                                        "ms": round(tm, 3), "steps": cst}
            del Ac, Ac0
        line["other_configs"] = others
        line["paper_context"] = {"Bulldozer64_K40c_n30720_nb512": "1092.4 GFLOP/s (Enhanced, no error, PAPER.md:374)",
                                 "Tardis_M2075_n20480_nb256": "268.7 GFLOP/s (PAPER.md:366)"}
    if rank == 0:
        print(json.dumps(line), flush=True)
    if dist:
        import torch.distributed as tdist
        P.abft_comm_destroy(comm)
        tdist.destroy_process_group()


if __name__ == "__main__":
    main()
