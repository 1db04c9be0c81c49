#!/usr/bin/env python
"""bench.py -- throughput of Neo's Hybrid key-switching hot path on B200.

Workload (BASELINE.json configs[1], Set-B of Table 4): N = 2^16, 36 Q limbs + 12 P
limbs of 36 bits, dnum = 3, level l = 35.  One STEP is one pass over every row of
SURVEY §8(a) for one batch of B ciphertexts per GPU:
    HMULT(ct_a, ct_b)  [tensor + KS(d2) + combine]  ->  Rescale          (a1, a3-a11)
    HROTATE(ct_c, g = 5)  [automorphism + KS + combine]                   (a2, a3-a10)
i.e. 2*B key-switches per step per GPU.  value = key-switches/s over all ranks (weak
scaling: every rank does its own B ciphertexts; data-parallel, no collective on the data
path).  Inputs are synthetic uniform residues (timing is data-independent; parity is
tested in tests/), resident in HBM, rotating over 2 input slots (216 MB at B=1) so that
inputs + the two 151 MB keys exceed the 126 MB L2.

`--impl reference` times the CPU oracle (oracle/, the reference arm of this tier) on the
same workload: each step is one Set-B key-switch on the host cores.
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

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "key-switch ops/s (HMult, HRot) at N=2^16 on 1/2/4/8 B200"
UNIT = "KS/s"
LOG_N, NUM_Q, NUM_P, DNUM, LEVEL = 16, 36, 12, 3, 35
HBM_FALLBACK = 6650.0   # GB/s, /opt/skills/guides/B200_PROFILING.md fallback


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=1000)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--batch", type=int, default=1, help="ciphertexts per GPU per step")
    ap.add_argument("--impl", choices=["neo", "reference"], default="neo")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-hoisted", action="store_true")
    ap.add_argument("--no-klss", action="store_true",
                    help="skip the KLSS vs Hybrid key-switch comparison at Set-C (SURVEY §8(f) row 1)")
    ap.add_argument("--fused-rescale", type=int, default=1, choices=[0, 1],
                    help="1: the step's HMULT -> Rescale is one neo_hmult_rescale call (bit-identical)")
    ap.add_argument("--no-latency", action="store_true", help="skip the per-operation latency distributions")
    ap.add_argument("--no-apps", action="store_true",
                    help="skip the application traces (HELR iteration, ResNet-20 layer; SURVEY §8(f) row 4)")
    ap.add_argument("--no-boot", action="store_true",
                    help="skip the bootstrapping timing (Set-B, 8 sparse slots; SURVEY §8(f) row 2)")
    ap.add_argument("--batch-hrot", type=int, default=256,
                    help="BASELINE configs[2]: this many independent HRot key-switches (one shared key) "
                         "split data-parallel over the ranks, plus a batch sweep up to it (0 = skip)")
    ap.add_argument("--streams", type=int, default=2, choices=[1, 2],
                    help="2: HRot runs on a second CUDA stream, overlapping HMult+Rescale")
    ap.add_argument("--graph", type=int, default=1, choices=[0, 1],
                    help="1: replay each step as a captured CUDA graph (the same ABI calls, captured once)")
    ap.add_argument("--chain-steps", type=int, default=1,
                    help="with 2 streams and graphs: one graph holds this many consecutive steps, each "
                         "stream running its chain of them back to back (one fork / join per graph "
                         "instead of per step); 1 = join after every step (the default: measured "
                         "4267 KS/s against 4162-4172 for 8-32 decoupled steps)")
    return ap.parse_args()


def workload_config(batch: int, world: int) -> dict:
    return {"workload": "setB_hmult_rescale_hrot", "N": 1 << LOG_N, "num_q": NUM_Q, "num_p": NUM_P,
            "dnum": DNUM, "level": LEVEL, "word_bits": 36, "batch_per_gpu": batch,
            "global_batch": batch * world, "ks_per_step_per_gpu": 2 * batch,
            "parallelism": f"dp{world}", "streams_per_gpu": 2,
            "l2": "inputs rotate over 2 slots (3 ciphertexts each) + 2 x 151 MB keys > 126 MB L2"}


# ----------------------------------------------------------------------------- inputs

def rand_limbs(moduli, seed, n):
    import synth
    return synth.uniform_residues(seed, moduli, n)


def rand_ct(moduli_q, seed, N, batch):
    return np.stack([np.stack([rand_limbs(moduli_q, seed + 7 * b + c, N) for c in range(2)])
                     for b in range(batch)])


def rand_evk(moduli, seed, N):
    return np.stack([np.stack([rand_limbs(moduli, seed + 2 * j + c, N) for c in range(2)])
                     for j in range(DNUM)])


# ----------------------------------------------------------------------------- clocks

class ClockSampler:
    """SM clock and clock-event (throttle) reasons sampled through NVML every ~2 ms in a
    thread (nvidia-smi's 100 ms period sees at most one sample of a 10 ms region).  The bench
    keeps the GPU under the same load after its timed region until the sampled window is
    >= 1 s long (`pad_until`), so `samples` counts the whole window and `samples_in_region`
    the timed region alone."""
    NAMES = (("hw_slowdown", "nvmlClocksEventReasonHwSlowdown"),
             ("hw_thermal_slowdown", "nvmlClocksEventReasonHwThermalSlowdown"),
             ("sw_thermal_slowdown", "nvmlClocksEventReasonSwThermalSlowdown"),
             ("sw_power_cap", "nvmlClocksEventReasonSwPowerCap"))

    def __init__(self, index: int, period_s: float = 0.002):
        self.index, self.period = index, period_s
        self.samples = []
        self.stop = threading.Event()
        self.h = None

    def __enter__(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            self.sm_max = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.masks = [(n, getattr(pynvml, m)) for n, m in self.NAMES]
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        except Exception as e:          # no NVML: report why instead of silently passing
            self.err = repr(e)
        return self

    def _run(self):
        nv, h = self.nv, self.h
        while not self.stop.is_set():
            try:
                sm = nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)
                rs = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                self.samples.append((time.monotonic(), sm, rs))
            except Exception:
                pass
            time.sleep(self.period)

    def wait_ready(self, timeout: float = 5.0):
        t0 = time.monotonic()
        while self.h is not None and not self.samples and time.monotonic() - t0 < timeout:
            time.sleep(0.001)
        self.t_begin = time.monotonic()

    def mark_end(self):
        self.t_end = time.monotonic()

    def window_s(self) -> float:
        return time.monotonic() - getattr(self, "t_begin", time.monotonic())

    def __exit__(self, *a):
        self.t_win_end = time.monotonic()
        self.stop.set()
        if self.h is not None:
            self.t.join(timeout=1)

    def summary(self) -> dict:
        if self.h is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0,
                    "error": getattr(self, "err", "NVML unavailable")}
        t0 = getattr(self, "t_begin", 0.0)
        t1 = getattr(self, "t_end", float("inf"))
        tw = getattr(self, "t_win_end", float("inf"))
        win = [x for x in self.samples if t0 <= x[0] <= tw]
        reg = [x for x in win if x[0] <= t1]
        reasons = sorted({n for _, _, rs in win for n, m in self.masks if rs & m})
        sm = [x[1] for x in win]
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": self.sm_max,
                "reasons": reasons, "samples": len(win), "samples_in_region": len(reg),
                "sm_mhz_in_region": statistics.median([x[1] for x in reg]) if reg else None,
                "window_s": round(tw - t0, 3), "source": "NVML every ~2 ms over the timed region, padded "
                "with the same untimed steps to a >= 1 s window"}


# ----------------------------------------------------------------------------- byte model

def bytes_model(batch: int, l: int = LEVEL, fused: bool = False) -> dict:
    """Algorithmic HBM bytes per step, per kernel kind, counted as SURVEY §8(d) counts them:
    one read plus one write of every limb an OPERATION transforms (limb = N residues of 8
    bytes; the NTT's two passes and their intermediate are not algorithmic traffic), plus the
    operands a fused epilogue reads.  Per key-switch at level l (Lq = l+1, P = 12, E = Lq + P,
    beta digits, up = beta*E - Lq ModUp outputs):
      NTT transforms: INTT(d) Lq + ModUp NTT up + INTT(acc_P) 2P + NTT(conv) 2Lq, each 2 limbs;
        the fused ModDown tail (a10) also reads acc_Q (2Lq) and the addend (HROT: sigma(c0),
        Lq; HMULT: d0, d1, 2Lq);
      BConv: ModUp reads Lq, writes up; ModDown reads 2P, writes 2Lq;
      KeyIP: reads d^ (beta*E), writes acc (2E), reads the key once per launch (2*beta*E limbs
        stored at 5 bytes per residue).
    Per step (HMULT+Rescale fused + HROT, B = 1, l = 35): 482 limb transforms + 250 tail
    operand limbs = 1214 limbs = 636.5 MB of NTT traffic (the fused HMULT+Rescale replaces the
    last NTT over Lq rows by one over l rows and adds the INTTs of acc_l, d_l: 4 transforms).
    tensor: reads a, b (4Lq), writes d0..d2 (3Lq); automorphism: c0 only (2Lq); elementwise: the
    fused Rescale's c_l kernel (reads acc_l, conv_l, d_l of both components, writes c_l: 8 limbs;
    the fold P*c_l itself is an operand of the next column pass, its 2 c_l limbs counted there)."""
    limb = (1 << LOG_N) * 8
    Lq, P = l + 1, NUM_P
    beta = -(-Lq // 12)
    E = Lq + P
    up = beta * E - Lq
    ks_tr = Lq + up + 2 * P                      # transforms up to the ModDown NTT
    hrot_tr, hrot_tail = ks_tr + 2 * Lq, 2 * Lq + Lq
    if fused:
        hm_tr, hm_tail = ks_tr + 4 + 2 * l, 2 * l + 2 * l + 2
        ew = batch * 8
        resc_tr, resc_tail = 0, 0
    else:
        hm_tr, hm_tail = ks_tr + 2 * Lq, 2 * Lq + 2 * Lq
        resc_tr, resc_tail = 2 + 2 * l, 2 * l
        ew = 0
    transforms = batch * (hrot_tr + hm_tr + resc_tr)
    ntt = 2 * transforms + batch * (hrot_tail + hm_tail + resc_tail)
    bconv = batch * 2 * ((Lq + up) + (2 * P + 2 * Lq))
    keyip = 2 * (batch * (beta * E + 2 * E) + 2 * beta * E * 5 / 8)
    tensor = batch * 7 * Lq
    auto = batch * 2 * Lq
    out = {"ntt": ntt, "bconv": bconv, "keyip": keyip, "combine": 0, "tensor": tensor, "automorphism": auto,
           "rescale_modswitch": 0, "rescale_combine": 0, "elementwise": ew}
    res = {k: v * limb for k, v in out.items()}
    res["_ntt_transforms"] = transforms
    return res


def merge_ntt(d: dict) -> dict:
    """neo_profile kinds with the two NTT passes merged into one kind 'ntt'."""
    out = {k: v for k, v in d.items() if k not in ("ntt_col", "ntt_row")}
    out["ntt"] = (d["ntt_col"][0] + d["ntt_row"][0], d["ntt_col"][1] + d["ntt_row"][1])
    return out


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return HBM_FALLBACK, "fallback (B200_PROFILING.md)"


def load_traffic(kind: str):
    """DRAM bytes (dram__bytes_read.sum + dram__bytes_write.sum) per launch of `kind` from the
    committed ncu --set full summary, next to that launch's algorithmic bytes, or None."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(p) as f:
            d = json.load(f)
        e = d.get(kind)
        if e is None:
            return None
        return {"bytes_per_launch": e["bytes_per_launch"], "algo_bytes_per_launch": e["algo_bytes_per_launch"],
                "ratio": round(e["bytes_per_launch"] / e["algo_bytes_per_launch"], 3), "launch": e["launch"],
                "source": e.get("source", "profiles/ncu_traffic.json")}
    except Exception:
        return None


def load_int8_peak():
    """The measured tcgen05 kind::i8 throughput at the NTT's MMA shape (M=128, N=80, K=32) and
    the best shape, from profiles/int8_peak.json (tools/i8peak.py)."""
    p = os.path.join(ROOT, "profiles", "int8_peak.json")
    try:
        with open(p) as f:
            d = json.load(f)
        shapes = d["tcgen05_i8_smem"]["shapes"]
        best = max(x["tops"] for x in shapes)
        n80 = [x["tops"] for x in shapes if x["N"] == 80]
        return {"tops": best, "tops_at_n80": n80[0] if n80 else None,
                "torch_int_mm_tops": max(x["tops"] for x in d.get("torch_int_mm", [{"tops": 0}])),
                "source": "profiles/int8_peak.json (tools/i8peak.py: tcgen05 kind::i8, operands in smem)"}
    except Exception:
        return None


# ----------------------------------------------------------------------------- CPU oracle

def oracle_keyswitch_rate(d, evk, budget_s=12.0, min_reps=1):
    """Time the CPU oracle (oracle/ckks.py fast mode) on Set-B key-switches."""
    from oracle import _core, ckks
    prm = ckks.set_b()
    reps, t0 = 0, time.perf_counter()
    while True:
        ckks.keyswitch(prm, d, LEVEL, evk)
        reps += 1
        el = time.perf_counter() - t0
        if reps >= min_reps and el >= budget_s:
            break
        if reps >= min_reps and el / reps * (reps + 1) > budget_s * 1.5:
            break
    return reps / el, reps, el, _core.lib().or_num_threads()


def host_cpu_info() -> dict:
    """nproc and the lscpu model name of the host the CPU baseline ran on."""
    model = None
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for ln in out.splitlines():
            if ln.lower().startswith("model name"):
                model = ln.split(":", 1)[1].strip()
                break
    except Exception:
        pass
    return {"nproc": os.cpu_count(), "lscpu_model": model}


def oracle_tiny_def_timing() -> dict:
    """SURVEY §8(d) config 1 leg: one HMULT + relinearise at the tiny config (N=2^12, 3 Q + 1 P,
    dnum=1) by the DEFINITIONAL oracle (O(N^2) NTT, Algorithm 1 BConv) on all host threads and
    on one thread (OpenMP thread count set through libgomp)."""
    import ctypes
    from oracle import _core, ckks
    import synth
    prm = ckks.tiny()
    ids = list(range(prm.num_q))
    ct = lambda sd: np.stack([synth.uniform_residues(sd + c, [prm.moduli[i] for i in ids], prm.N) for c in range(2)])
    allids = list(range(prm.num_q + prm.num_p))
    evk = np.stack([np.stack([synth.uniform_residues(70 + 2 * j + c, [prm.moduli[i] for i in allids], prm.N)
                              for c in range(2)]) for j in range(prm.dnum)])
    a, b = ct(1), ct(3)
    L = _core.lib()
    gomp = ctypes.CDLL("libgomp.so.1")
    full = L.or_num_threads()
    res = {"op": "one HMULT + relinearise, tiny config, mode=def", "nproc": os.cpu_count()}
    for name, nt in (("all_threads", full), ("one_thread", 1)):
        gomp.omp_set_num_threads(nt)
        t0 = time.perf_counter()
        ckks.hmult(prm, a, b, prm.max_level, evk, mode="def")
        res[name] = {"threads": nt, "seconds": round(time.perf_counter() - t0, 3)}
    gomp.omp_set_num_threads(full)
    return res


# ----------------------------------------------------------------------------- reference arm

def run_reference(args):
    """The reference arm: the CPU oracle, as it stands, on the host cores (rank 0 only).  A
    Set-B key-switch takes ~1 s there, so a step is one of its six stages in order -- INTT of d;
    ModUp + NTT + KeyIP of digit 0, 1, 2; ModDown of component 0, 1 (oracle/ckks.keyswitch's a3-a10,
    the same calls) -- and six steps make one key-switch: value = steps / 6 / time (KS/s), so any
    --steps K finishes in minutes."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import numpy as np
    from oracle import _core, ckks
    prm = ckks.set_b()
    N = prm.N
    d = rand_limbs(prm.q, 0x4E454F, N)
    evk = rand_evk(prm.moduli, 0x4E454F + 100, N)
    q_ids = list(range(LEVEL + 1))
    p_ids = prm.p_ids
    ext = q_ids + p_ids
    pos = {t: k for k, t in enumerate(ext)}
    digits = prm.digits(LEVEL)
    pinv = [pow(prm.P % prm.moduli[i], -1, prm.moduli[i]) for i in q_ids]
    st = {}

    def stage(k):
        if k == 0:                                             # a3
            st["coef"] = ckks.intt(prm, d, q_ids)
            st["acc"] = np.zeros((2, len(ext), N), dtype=np.uint64)
        elif k <= 3:                                           # a4-a6 for digit k-1
            dj = digits[k - 1]
            targets = [t for t in ext if t not in dj]
            up = ckks.ntt(prm, ckks.bconv(prm, st["coef"][dj[0]:dj[-1] + 1], dj, targets), targets)
            dhat = np.empty((len(ext), N), dtype=np.uint64)
            for t in dj:
                dhat[pos[t]] = d[t]
            for i, t in enumerate(targets):
                dhat[pos[t]] = up[i]
            for c in range(2):
                st["acc"][c] = ckks.add(prm, st["acc"][c], ckks.mul(prm, dhat, evk[k - 1, c][ext], ext), ext)
        else:                                                  # a7-a10 for component k-4
            acc = st["acc"][k - 4]
            acc_p = ckks.intt(prm, acc[[pos[t] for t in p_ids]], p_ids)
            conv = ckks.ntt(prm, ckks.bconv(prm, acc_p, p_ids, q_ids), q_ids)
            st[f"out{k - 4}"] = ckks.scalar_mul(prm, ckks.sub(prm, acc[: LEVEL + 1], conv, q_ids), pinv, q_ids)

    for w in range(args.warmup):
        stage(w % 6)
    t0 = time.perf_counter()
    for k in range(args.steps):
        stage(k % 6)
    el = time.perf_counter() - t0
    v = args.steps / 6 / el
    cores = _core.lib().or_num_threads()
    line = {"metric": METRIC, "value": v, "unit": UNIT, "impl": "reference", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * el / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u64",
            "data": "synthetic", "config": workload_config(1, 1),
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle",
                             "sample": "each step = one of the six stages of a Set-B key-switch (l=35, B=1) by "
                                       "the CPU oracle (INTT; ModUp+NTT+KeyIP of digit 0/1/2; ModDown of c0/c1); "
                                       "6 steps = 1 key-switch"},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    emit(line)


# ----------------------------------------------------------------------------- neo arm

def graph_capture(fn, side=None):
    """Capture fn() (a sequence of C-ABI calls on the current stream) as a CUDA graph on a side
    stream after one eager warm-up there.  Returns (graph, output of the captured call) or
    (None, None) when capture fails (the caller then times eagerly)."""
    import torch
    try:
        side = torch.cuda.Stream() if side is None else side
        side.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(side):
            fn()
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=side):
                out = fn()
        torch.cuda.current_stream().wait_stream(side)
        torch.cuda.synchronize()
        return g, out
    except Exception as exc:
        print(f"graph capture failed ({exc}); timing eagerly", file=sys.stderr)
        torch.cuda.synchronize()
        return None, None


def _same(a, b) -> bool:
    import torch
    return torch.equal(a.view(torch.int64), b.view(torch.int64))


def run_neo(args):
    import torch
    import torch.distributed as dist
    from paper_conf_isca_jiaodwfcm0z25_b200 import neo

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # NEO_BENCH_BACKEND=gloo runs several ranks on one GPU (a functional check of the N > 1
    # paths on a 1-GPU box; not a measurement).  The driver's runs use NCCL, one GPU per rank.
    backend = os.environ.get("NEO_BENCH_BACKEND", "nccl")
    if backend != "nccl":
        local = local % torch.cuda.device_count()
    torch.cuda.set_device(local)
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)

    def barrier():
        if world > 1:
            dist.barrier()

    def agree(ok: bool) -> bool:
        """True on every rank iff true on all ranks (keeps the ranks' collectives in step when
        something optional -- a graph capture -- succeeded on some ranks only)."""
        if world == 1:
            return ok
        t = torch.tensor([1.0 if ok else 0.0], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MIN)
        return bool(t.item() > 0.5)

    B = args.batch
    ctx = neo.Context(LOG_N, NUM_Q, NUM_P, DNUM, device=local)
    N, Lq = ctx.N, LEVEL + 1
    seed = 0x4E454F + 1000 * rank
    relin_np = rand_evk(ctx.moduli, seed + 100, N)
    rot_np = rand_evk(ctx.moduli, seed + 200, N)
    relin = neo.EvalKey(ctx, torch.from_numpy(relin_np).cuda())
    rot = neo.EvalKey(ctx, torch.from_numpy(rot_np).cuda())
    qmods = ctx.q[:Lq]
    SLOTS = 2
    host_in = [[rand_ct(qmods, seed + 10 * s + k, N, B) for k in range(3)] for s in range(SLOTS)]
    dev_in = [[torch.from_numpy(x).cuda() for x in slot] for slot in host_in]
    def new_outs():
        return (torch.empty((B, 2, Lq, N), dtype=torch.uint64, device="cuda"),
                torch.empty((B, 2, LEVEL, N), dtype=torch.uint64, device="cuda"),
                torch.empty((B, 2, Lq, N), dtype=torch.uint64, device="cuda"))
    hm_o, rs_o, hr_o = new_outs()
    ws_n = max(ctx.workspace_size(neo.NEO_OP_HMULT, LEVEL, B), ctx.workspace_size(neo.NEO_OP_HROT, LEVEL, B),
               ctx.workspace_size(neo.NEO_OP_RESCALE, LEVEL, B), ctx.workspace_size(neo.NEO_OP_HMULT_RESCALE, LEVEL, B))
    ws = torch.empty(ws_n // 8, dtype=torch.uint64, device="cuda")
    ws2 = torch.empty(ws_n // 8, dtype=torch.uint64, device="cuda") if args.streams == 2 else ws
    main_st = torch.cuda.current_stream()
    side_st = torch.cuda.Stream() if args.streams == 2 else main_st
    ev_go, ev_done = torch.cuda.Event(), torch.cuda.Event()
    g = 5                                   # 5^1 mod 2N: rotate slots left by one

    launches = [0]

    def step(s, a=None, b=None, c=None, two=None, outs=None, fork=True, join=True):
        """HMult -> Rescale on the current stream; HRot (independent ciphertext) on the side
        stream (two=True), joined back into the current stream before the step ends (join) or,
        inside a multi-step graph, only after the last step of the graph."""
        two = (args.streams == 2) if two is None else two
        a = dev_in[s][0] if a is None else a
        b = dev_in[s][1] if b is None else b
        c = dev_in[s][2] if c is None else c
        hm_out, rs_out, hr_out = outs if outs is not None else (hm_o, rs_o, hr_o)
        main = torch.cuda.current_stream()
        side = side_st if two else main
        if two and fork:
            ev_go.record(main)
            side.wait_event(ev_go)
        neo.neo_hrot(ctx, rot, g, c, LEVEL, hr_out, B, ws2 if two else ws, stream=side)
        n = neo.last_launch_count()
        if args.fused_rescale:          # Rescale(HMULT) in one call, bit-identical to the pair
            neo.neo_hmult_rescale(ctx, relin, a, b, LEVEL, rs_out, B, ws, stream=main)
            n += neo.last_launch_count()
        else:
            neo.neo_hmult(ctx, relin, a, b, LEVEL, hm_out, B, ws, stream=main)
            n += neo.last_launch_count()
            neo.neo_rescale(ctx, hm_out, LEVEL, rs_out, B, ws, stream=main)
            n += neo.last_launch_count()
        if two and join:
            ev_done.record(side)
            main.wait_event(ev_done)
        launches[0] += n
        return n

    # warm-up (untimed)
    for w in range(max(args.warmup, 1)):
        step(w % SLOTS)
    torch.cuda.synchronize()
    barrier()
    torch.cuda.synchronize()

    # optional CUDA graphs: one captured step per input slot (same ABI calls, captured once)
    graphs = None
    if args.graph:
        graphs = []
        for sl in range(SLOTS):
            gr = torch.cuda.CUDAGraph()
            with torch.cuda.graph(gr):
                n_per_step = step(sl)
            graphs.append(gr)
        for w in range(2):
            graphs[w % SLOTS].replay()
        torch.cuda.synchronize()

    # multi-step graphs: CH consecutive steps with one fork / join, so each stream runs its chain
    # of the CH steps back to back (the steps are independent: own inputs, per-stream workspaces)
    CH = max(1, args.chain_steps) if (graphs is not None and args.streams == 2) else 1
    if CH > 1 and CH % SLOTS:
        CH += SLOTS - CH % SLOTS
    multi = None
    if CH > 1:
        multi = torch.cuda.CUDAGraph()
        with torch.cuda.graph(multi):
            for i in range(CH):
                step(i % SLOTS, fork=(i == 0), join=(i == CH - 1))
        for _ in range(2):
            multi.replay()
        torch.cuda.synchronize()

    def run_steps(k0, n):
        """steps k0 .. k0+n-1: whole multi-step graphs where they fit (k0 on a graph boundary)"""
        k = k0
        while k < k0 + n:
            if multi is not None and k % CH == 0 and k + CH <= k0 + n:
                multi.replay()
                launches[0] += CH * n_per_step
                k += CH
            elif graphs is not None:
                graphs[k % SLOTS].replay()
                launches[0] += n_per_step
                k += 1
            else:
                step(k % SLOTS)
                k += 1

    def run_step(k):
        run_steps(k, 1)

    # timed region A (the headline): device time with CUDA events on the launching stream
    launches[0] = 0
    t_start, t_end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        clk.wait_ready()
        barrier()
        torch.cuda.synchronize()
        t_start.record()
        run_steps(0, args.steps)
        t_end.record()
        torch.cuda.synchronize()
        clk.mark_end()
        gpu_launches = launches[0]
        # keep the same load (untimed) until the clock window is >= 1 s long
        k = args.steps
        while clk.window_s() < 1.0:
            run_steps(k, 48)
            k += 48
            torch.cuda.synchronize()
    barrier()
    torch.cuda.synchronize()
    ms = t_start.elapsed_time(t_end)
    if world > 1:
        t = torch.tensor([ms], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    ms_step = ms / args.steps
    value = 2 * B * world / (ms_step / 1e3)

    # timed region B: the same K steps on ONE stream, every kernel bracketed by CUDA events on
    # its stream (neo_profile_enable) -> per-kernel durations, shares and the roofline
    neo.neo_profile_enable(True)
    p_start, p_end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    p_start.record()
    for k in range(args.steps):
        step(k % SLOTS, two=False)
    p_end.record()
    torch.cuda.synchronize()
    prof = merge_ntt(neo.neo_profile_read())
    neo.neo_profile_enable(False)
    ms_step_1s = p_start.elapsed_time(p_end) / args.steps

    # roofline of the dominant kernel kind (SURVEY §8(d) bytes; the NTT's two passes as one kind)
    peak, peak_src = load_peaks()
    bm = bytes_model(B, fused=bool(args.fused_rescale))
    n_transforms = bm.pop("_ntt_transforms")
    step_ms = {k: v[0] / args.steps for k, v in prof.items()}
    ms_step_ref = ms_step_1s
    dom = max(step_ms, key=lambda k: step_ms[k])
    n_launch_dom = prof[dom][1] / args.steps
    achieved = bm[dom] / (step_ms[dom] / 1e3) / 1e9 if step_ms[dom] > 0 else None
    traffic = load_traffic(dom)
    ntt_impl = "tc" if ctx.ntt_impl == neo.NEO_NTT_TC else "fp64"
    # second roofline of the NTT: int8 tensor-core work against the measured tcgen05 i8 peak
    # (profiles/int8_peak.json) for the tcgen05 form -- per limb transform 2 passes x 2 stages x
    # 12 MMAs of 128 x 80 x 32 per 16-transform tile = 1920 MACs per coefficient -- or FP64
    # operations against 63 DFMA-pipe ops/clk/SM for the CUDA-core form
    alt = None
    i8 = load_int8_peak()
    try:
        mhz = float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["sm_max_mhz"])
    except Exception:
        mhz = 1965.0
    if ntt_impl == "tc":
        ops = 2.0 * 1920 * (1 << LOG_N) * n_transforms
        ach = ops / (step_ms["ntt"] / 1e3) if step_ms["ntt"] > 0 else 0.0
        alt = {"bound": "tensor", "kernel": "ntt", "dtype": "u8xu8->s32", "achieved": ach / 1e12,
               "peak": i8["tops"] if i8 else None, "unit": "TOP/s",
               "frac": ach / 1e12 / i8["tops"] if i8 else None, "ops_per_step": ops,
               "peak_source": i8["source"] if i8 else "not measured"}
    else:
        fw, iv = (358, 124) if args.fused_rescale else (430, 122)
        ops = (fw * (45.4 + 30.8) + iv * (48.4 + 27.8)) * (1 << LOG_N) * B
        pk = 63 * torch.cuda.get_device_properties(local).multi_processor_count * mhz * 1e6
        ach = ops / (step_ms["ntt"] / 1e3) if step_ms["ntt"] > 0 else 0.0
        alt = {"bound": "fp64", "kernel": "ntt", "achieved": ach / 1e12, "peak": pk / 1e12, "unit": "Tops/s",
               "frac": ach / pk, "ops_per_step": ops}
    breakdown = {k: {"ms_per_step": round(step_ms[k], 5), "launches_per_step": prof[k][1] / args.steps,
                     "share": round(step_ms[k] / ms_step_ref, 4) if ms_step_ref > 0 else None,
                     "algo_GBps": round(bm[k] / (step_ms[k] / 1e3) / 1e9, 1) if step_ms[k] > 0 else None,
                     "frac_hbm": round(bm[k] / (step_ms[k] / 1e3) / 1e9 / peak, 4) if step_ms[k] > 0 else None}
                 for k in step_ms}

    # per-operation latency at Set-B (l = 35, B = 1) -- median / p10 / p90
    # of 100 single calls, each bracketed by CUDA events on the calling stream after 10 warm-ups;
    # "warm": the same inputs back to back; "flushed": a 256 MB buffer (> the 126 MB L2) is
    # overwritten before every call.  Context: the paper's Table 6 (A100, Set-C): HMult 3472.5 us,
    # HRotate 3422.1 us, Rescale 114.3 us, PMult 81.7 us, HAdd 46.1 us.
    latency = None
    if not args.no_latency:
        a_, b_, c_ = dev_in[0]
        o1, o2, o3 = new_outs()
        flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
        d_ks = a_[:, 1].contiguous()
        k0_, k1_ = torch.empty_like(d_ks), torch.empty_like(d_ks)
        ops_ = {
            "keyswitch": lambda: neo.neo_keyswitch(ctx, relin, d_ks, LEVEL, k0_, k1_, B, ws),
            "hmult": lambda: neo.neo_hmult(ctx, relin, a_, b_, LEVEL, o1, B, ws),
            "hmult_rescale": lambda: neo.neo_hmult_rescale(ctx, relin, a_, b_, LEVEL, o2, B, ws),
            "hrot": lambda: neo.neo_hrot(ctx, rot, g, c_, LEVEL, o3, B, ws),
            "rescale": lambda: neo.neo_rescale(ctx, o1, LEVEL, o2, B, ws),
        }
        latency = {"config": "Set-B l=35, B=1, one call per sample", "unit": "us",
                   "paper_context_table6_a100_setc_us": {"hmult": 3472.5, "hrot": 3422.1, "rescale": 114.3}}
        for name, fn in ops_.items():
            res = {}
            for mode in ("warm", "flushed"):
                for _ in range(10):
                    fn()
                torch.cuda.synchronize()
                samples = []
                for _ in range(100):
                    if mode == "flushed":
                        flush.fill_(1)
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record()
                    fn()
                    e1.record()
                    e1.synchronize()
                    samples.append(e0.elapsed_time(e1) * 1e3)
                samples.sort()
                res[mode] = {"median": round(samples[50], 1), "p10": round(samples[10], 1),
                             "p90": round(samples[90], 1)}
            latency[name] = res
        del flush

    # one Set-B key-switch (l = 35, B = 1) limb-sharded over all
    # ranks (round-robin limbs; two all-gathers, NCCL when N > 1), eager; at N = 1 the same code
    # path on one rank.  Latency = the slowest rank's CUDA-event time per key-switch.
    sharded_ks = None
    if not args.no_latency:
        from paper_conf_isca_jiaodwfcm0z25_b200.sharded import NeoOps, ShardPlan, limb_sharded_keyswitch
        plan = ShardPlan(LEVEL, NUM_Q, NUM_P, ctx.alpha, world, rank, strided=True)
        sops = NeoOps(ctx)
        d_loc = dev_in[0][0][:, 1].contiguous().view(torch.int64)[:, plan.my_q].contiguous().view(torch.uint64)
        for _ in range(3):
            limb_sharded_keyswitch(sops, plan, d_loc, relin)
        torch.cuda.synchronize()
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(20):
            limb_sharded_keyswitch(sops, plan, d_loc, relin)
        e1.record()
        torch.cuda.synchronize()
        sks = e0.elapsed_time(e1) / 20
        if world > 1:
            t = torch.tensor([sks], dtype=torch.float64, device="cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            sks = float(t.item())
        sharded_ks = {"ranks": world, "ms_per_keyswitch": round(sks, 4), "unit": "ms",
                      "limbs_per_rank": len(plan.mine),
                      "note": "eager Python orchestration over C-ABI building blocks (host-issued launches)"}

    # the same key-switch through the NATIVE limb-sharded call (neo_keyswitch_sharded: both
    # exchanges inside the library, NCCL over NVLink for N > 1, per-digit gathers overlapped with
    # the previous digit's BConv + NTT), eager and as a captured CUDA graph
    sharded_native = None
    ncomm, comm_err = None, None
    if not args.no_latency:
        try:
            if world > 1:
                uid = torch.zeros(128, dtype=torch.uint8, device="cuda")
                if rank == 0:
                    uid.copy_(torch.frombuffer(bytearray(neo.Comm.unique_id()), dtype=torch.uint8))
                dist.broadcast(uid, src=0)
                ncomm = neo.Comm.create(ctx, bytes(uid.cpu().numpy().tobytes()), world, rank)
            else:
                ncomm = neo.Comm.create(ctx, bytes(128), 1, 0)
        except neo.NeoError as e:       # e.g. several ranks on one GPU (NEO_BENCH_BACKEND=gloo): NCCL refuses
            ncomm, comm_err = None, str(e)[:200]
        if not agree(ncomm is not None):
            if ncomm is not None:
                ncomm.close()
                ncomm = None
            sharded_native = {"ranks": world, "unavailable": comm_err or "the communicator failed on another rank"}
    if ncomm is not None:
        nq_ids, _ = ncomm.limbs(LEVEL)
        full_d = dev_in[0][0][:, 1].contiguous()
        dl = full_d.view(torch.int64)[:, nq_ids].contiguous().view(torch.uint64) if nq_ids else None
        so0 = torch.empty((B, len(nq_ids), N), dtype=torch.uint64, device="cuda") if nq_ids else None
        so1 = torch.empty_like(so0) if nq_ids else None
        sws = ncomm.workspace(LEVEL, B)
        run_native = lambda: neo.neo_keyswitch_sharded(ctx, ncomm, relin, dl, LEVEL, so0, so1, B, sws)
        for _ in range(3):
            run_native()
        torch.cuda.synchronize()
        barrier()

        def time_native(fn, reps=20):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(reps):
                fn()
            e1.record()
            torch.cuda.synchronize()
            v = e0.elapsed_time(e1) / reps
            if world > 1:
                t = torch.tensor([v], dtype=torch.float64, device="cuda")
                dist.all_reduce(t, op=dist.ReduceOp.MAX)
                v = float(t.item())
            return v
        eager_ms = time_native(run_native)
        graph_ms = None
        try:
            gr = torch.cuda.CUDAGraph()
            with torch.cuda.graph(gr):
                run_native()
            graph_ms = time_native(gr.replay)
        except Exception as e:          # noqa: BLE001 -- reported in the line
            graph_ms = f"capture failed: {e!r}"[:200]
        sharded_native = {"ranks": world, "unit": "ms", "ms_per_keyswitch_eager": round(eager_ms, 4),
                          "ms_per_keyswitch_graph": round(graph_ms, 4) if isinstance(graph_ms, float) else graph_ms,
                          "q_limbs_per_rank": len(nq_ids), "transport": "nccl" if world > 1 else "none (1 rank)",
                          "note": "neo_keyswitch_sharded (native C-ABI); slowest rank, CUDA events"}
        ncomm.close()

    # secondary: hoisted rotations (one ModUp shared by n_rot rotations of the same ciphertext)
    hoisted = None
    if not args.no_hoisted:
        n_rot = 4
        hk = []
        for r in range(n_rot):
            gr = pow(5, r + 1, 2 * N)
            hk.append(neo.EvalKey(ctx, torch.from_numpy(rand_evk(ctx.moduli, seed + 300 + 7 * r, N)).cuda(),
                                  hoisted_galois=gr))
        hout = torch.empty((n_rot, B, 2, Lq, N), dtype=torch.uint64, device="cuda")
        hws = ctx.workspace(neo.NEO_OP_HROT_HOISTED, LEVEL, B)
        for w in range(3):
            neo.neo_hrot_hoisted(ctx, hk, dev_in[w % SLOTS][2], LEVEL, hout, B, hws)
        torch.cuda.synchronize()
        h0, h1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        kh = max(3, min(args.steps, 100))
        h0.record()
        for k in range(kh):
            neo.neo_hrot_hoisted(ctx, hk, dev_in[k % SLOTS][2], LEVEL, hout, B, hws)
        h1.record()
        torch.cuda.synchronize()
        hms = h0.elapsed_time(h1) / kh
        hoisted = {"n_rot": n_rot, "value": n_rot * B * world / (hms / 1e3), "unit": "rotations/s",
                   "ms_per_call": hms, "note": "neo_hrot_hoisted, one stream, Set-B l=35"}
        del hk

    # BASELINE configs[2]: a batch of `batch_hrot` independent HRot(g=5)
    # key-switches sharing one rotation key, split data-parallel over the ranks (weak per-rank
    # shard, no collective), plus the Fig. 17 analogue: the same call at smaller batches.
    # Timing is data-independent; inputs are uniform residues < 2^35 (< every 36-bit q), made
    # on the device.
    batch_block = None
    if args.batch_hrot > 0:
        Bg = args.batch_hrot
        Bl = max(1, Bg // world)
        gen = torch.Generator(device="cuda")
        gen.manual_seed(seed + 77)
        big_in = torch.randint(0, 1 << 35, (Bl, 2, Lq, N), dtype=torch.int64, device="cuda",
                               generator=gen).view(torch.uint64)
        big_out = torch.empty_like(big_in)
        big_ws = torch.empty(ctx.workspace_size(neo.NEO_OP_HROT, LEVEL, Bl) // 8, dtype=torch.uint64, device="cuda")
        sweep = []
        sizes = sorted({b for b in (8, 16, 32, 64, 128) if b < Bl} | {Bl})
        for bs in sizes:
            neo.neo_hrot(ctx, rot, g, big_in[:bs], LEVEL, big_out[:bs], bs, big_ws)          # warm-up
            torch.cuda.synchronize()
            barrier()
            reps = 3
            b0, b1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            b0.record()
            for _ in range(reps):
                neo.neo_hrot(ctx, rot, g, big_in[:bs], LEVEL, big_out[:bs], bs, big_ws)
            b1.record()
            torch.cuda.synchronize()
            bms = b0.elapsed_time(b1) / reps
            if world > 1:
                t = torch.tensor([bms], dtype=torch.float64, device="cuda")
                dist.all_reduce(t, op=dist.ReduceOp.MAX)
                bms = float(t.item())
            sweep.append({"batch_per_gpu": bs, "ms_per_call": round(bms, 4),
                          "value": bs * world / (bms / 1e3)})
        last = sweep[-1]
        batch_block = {"config": "BASELINE configs[2]: N=2^16, L=35, dnum=3, batch of independent HRot "
                                 "key-switches (one shared key), data-parallel over the GPUs",
                       "global_batch": Bl * world, "batch_per_gpu": Bl, "value": last["value"], "unit": "HRot/s",
                       "ms_per_call": last["ms_per_call"], "sweep": sweep,
                       "timing": "CUDA events around 3 neo_hrot calls per size after 1 warm-up, max over ranks"}
        del big_in, big_out, big_ws
        torch.cuda.empty_cache()

    # SURVEY §8(f) row 1 (Table 8 / Fig. 16 analogue): one key-switch at Set-C (N=2^16, L=35,
    # dnum=9, alpha~=5) with the KLSS key at WordSize_T = 48 (Table 4 as printed, L511: 8 T primes)
    # and at WordSize_T = 36 (10 T primes), and with the Hybrid key of the same parameters, B = 1
    # and B = 8 per GPU, CUDA events, max over ranks.  Keys and inputs are uniform residues < 2^35
    # made on the device (timing is data-independent).
    klss_block = None
    if not args.no_klss:
        gen = torch.Generator(device="cuda")
        gen.manual_seed(seed + 91)
        rnd = lambda *shape: torch.randint(0, 1 << 35, shape, dtype=torch.int64, device="cuda",
                                           generator=gen).view(torch.uint64)
        bt = -(-(36 + 4) // 5)
        ctxs = {48: neo.Context(16, 36, 4, 9, alpha_t=5, word_bits_t=48, device=local),
                36: neo.Context(16, 36, 4, 9, alpha_t=5, device=local)}
        keys = {"klss_t48": (ctxs[48], neo.EvalKey(ctxs[48], rnd(2, bt, 9, ctxs[48].alpha_p, N), klss=True)),
                "klss_t36": (ctxs[36], neo.EvalKey(ctxs[36], rnd(2, bt, 9, ctxs[36].alpha_p, N), klss=True)),
                "hybrid": (ctxs[48], neo.EvalKey(ctxs[48], rnd(9, 2, 40, N)))}
        klss_block = {"config": "Set-C (Table 4): N=2^16, L=35, dnum=9, alpha~=5, level 35; KLSS with "
                                f"WordSize_T=48 (alpha'={ctxs[48].alpha_p}) and 36 (alpha'={ctxs[36].alpha_p})",
                      "unit": "KS/s", "timing": "CUDA events around 20 neo_keyswitch calls after 3 warm-ups"}
        for Bk in (1, 8):
            dk = rnd(Bk, Lq, N)
            o0, o1 = torch.empty_like(dk), torch.empty_like(dk)
            for meth, (cctx, key) in keys.items():
                wsk = torch.empty(cctx.workspace_size(neo.NEO_OP_KEYSWITCH, LEVEL, Bk) // 8, dtype=torch.uint64,
                                  device="cuda")
                for _ in range(3):
                    neo.neo_keyswitch(cctx, key, dk, LEVEL, o0, o1, Bk, wsk)
                torch.cuda.synchronize()
                barrier()
                k0, k1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                k0.record()
                for _ in range(20):
                    neo.neo_keyswitch(cctx, key, dk, LEVEL, o0, o1, Bk, wsk)
                k1.record()
                torch.cuda.synchronize()
                kms = k0.elapsed_time(k1) / 20
                if world > 1:
                    t = torch.tensor([kms], dtype=torch.float64, device="cuda")
                    dist.all_reduce(t, op=dist.ReduceOp.MAX)
                    kms = float(t.item())
                klss_block[f"{meth}_B{Bk}"] = {"ms_per_call": round(kms, 4), "value": Bk * world / (kms / 1e3)}
                del wsk
            del dk, o0, o1
        del keys
        for cctx in ctxs.values():
            cctx.close()
        torch.cuda.empty_cache()

    # SURVEY §8(f) row 2 / BASELINE metric "bootstrap ms": one sparse-slot bootstrapping
    # (paper_conf_isca_jiaodwfcm0z25_b200.boot: ModRaise, SubSum, CoeffToSlot, EvalMod,
    # SlotToCoeff; n = 8 slots, r = 12 squarings, 20 levels) at Set-B on every rank (DP).  Keys
    # and plaintext constants are uniform residues made on the device (timing is data-independent;
    # correctness: tests/test_gpu_boot.py).
    boot_block = None
    if not args.no_boot:
        from paper_conf_isca_jiaodwfcm0z25_b200 import boot as gboot
        from paper_conf_isca_jiaodwfcm0z25_b200.sharded_boot import ShardedBootstrapper
        gen = torch.Generator(device="cuda")
        gen.manual_seed(seed + 123)
        rnd = lambda *shape: torch.randint(0, 1 << 35, shape, dtype=torch.int64, device="cuda",
                                           generator=gen).view(torch.uint64)
        evk_b = rnd(DNUM, 2, NUM_Q + NUM_P, N)          # one random key serves every Galois element
        bct = rnd(1, 2, 1, N)

        def time_runs(run, reps):
            barrier()
            b0, b1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            b0.record()
            for _ in range(reps):
                run()
            b1.record()
            torch.cuda.synchronize()
            t_ = b0.elapsed_time(b1) / reps
            if world > 1:
                t = torch.tensor([t_], dtype=torch.float64, device="cuda")
                dist.all_reduce(t, op=dist.ReduceOp.MAX)
                t_ = float(t.item())
            return t_

        def boot_case(nb, rb, fl, sharded, boost=(0, 0), ds_sq=0):
            """Time one bootstrap configuration: eager and as a CUDA-graph replay (output checked
            equal), and optionally the limb-sharded form over all ranks (graph, NCCL)."""
            keys = {"relin": neo.EvalKey(ctx, evk_b)}
            for gg in gboot.rotations(N, nb, fl):
                keys[gg] = neo.EvalKey(ctx, evk_b)
            for gg in gboot.hoisted_rotations(N, nb, fl):
                keys[("h", gg)] = neo.EvalKey(ctx, evk_b, hoisted_galois=gg)
            consts = {k: rnd(l + 1, N) for k, l in gboot.const_levels(LEVEL, nb, rb, N, fl, boost, ds_sq).items()}
            bt = gboot.Bootstrapper(ctx, nb, rb, keys, consts, fft_levels=fl, boost=boost, ds_sq=ds_sq)
            for _ in range(2):
                bt.run(bct)
            torch.cuda.synchronize()
            eager = time_runs(lambda: bt.run(bct), 3)
            ref_out = bt.run(bct)[0].clone()
            bgraph, bg_out = graph_capture(lambda: bt.run(bct)[0])
            gms = None
            if not agree(bgraph is not None):
                bgraph = None
            if bgraph is not None:
                bgraph.replay()
                torch.cuda.synchronize()
                assert _same(bg_out, ref_out), "graph replay of the bootstrap differs from the eager run"
                gms = time_runs(bgraph.replay, 5)
            best = gms if gms is not None else eager
            out = {"ms_per_bootstrap": round(best, 3), "value": world / (best / 1e3), "unit": "bootstraps/s",
                   "graph": gms is not None, "ms_eager": round(eager, 3),
                   "levels": f"{LEVEL} -> {LEVEL - gboot.levels_used(rb, fl, boost, ds_sq)}", "boost": list(boost),
                   "ds_squarings": ds_sq,
                   "rotation_keys": len(gboot.rotations(N, nb, fl)) + len(gboot.hoisted_rotations(N, nb, fl))}
            if sharded:
                # config 4's multi-GPU form: the same bootstrap limb-sharded over all ranks
                # (round-robin limbs; two all-gathers per key-switch, one limb broadcast per
                # Rescale; NCCL).  At N = 1 the sharded code path runs on one rank.
                sbt = ShardedBootstrapper(ctx, nb, rb, keys, consts, world, rank, fft_levels=fl, boost=boost, ds_sq=ds_sq)
                sct0 = sbt.shard(bct, 0)
                sref = sbt.run(sct0)[0].clone()
                # graph capture only on one rank: a capture that failed on some ranks mid-way
                # through NCCL collectives could desynchronise them; with N > 1 the exchanges
                # are timed eagerly (host-issued)
                sgraph = sg_out = sbt_g = None
                if world == 1:
                    s_side = torch.cuda.Stream()
                    sbt_g = ShardedBootstrapper(ctx, nb, rb, keys, consts, world, rank, stream=s_side, fft_levels=fl,
                                                boost=boost, ds_sq=ds_sq)
                    sgraph, sg_out = graph_capture(lambda: sbt_g.run(sct0)[0], side=s_side)
                if sgraph is not None:
                    sgraph.replay()
                    torch.cuda.synchronize()
                    assert _same(sg_out, sref), "graph replay of the sharded bootstrap differs from the eager run"
                sms = time_runs(sgraph.replay if sgraph is not None else (lambda: sbt.run(sct0)), 3)
                out["limb_sharded"] = {
                    "ranks": world, "ms_per_bootstrap": round(sms, 3), "value": 1 / (sms / 1e3),
                    "unit": "bootstraps/s", "graph": sgraph is not None,
                    "exchanges": "per key-switch 2 all-gathers (Q limbs before ModUp, P limbs before ModDown); "
                                 "per Rescale / ModRaise 1 broadcast of one limb (2 rows)"}
                del sbt, sbt_g, sgraph
            del keys, consts, bt, bgraph
            torch.cuda.empty_cache()
            return out

        full = boot_case(N // 2, 9, 4, sharded=True, boost=(20, 20), ds_sq=4)     # oracle.boot.set_b_full()
        sparse = boot_case(8, 9, 0, sharded=False, boost=(20, 20), ds_sq=4)    # oracle.boot.set_b()
        boot_block = dict(full, config="Set-B (N=2^16, L=35, dnum=3), full slots (32768), r=9 squarings (4 at ~q^2 scale, Double Rescale), "
                                       "CoeffToSlot / SlotToCoeff as 4 special-FFT BSGS levels each (stages 4-4-4-3)",
                          timing="CUDA events around 5 graph replays (3 eager runs) after warm-ups, max over "
                                 "ranks; replay output checked equal to the eager run; keys / constants synthetic",
                          sparse_8_slots=sparse)
        del evk_b

    # SURVEY §8(f) row 4 / BASELINE configs[4]: the application traces (reading APP,
    # paper_conf_isca_jiaodwfcm0z25_b200.apps) at Set-B on every rank (DP): one HELR iteration
    # over 1,024 samples of 196 -> 256 features (8 ciphertexts of 128 x 256, L530) and one
    # ResNet-20 convolution layer (16 channels of 32 x 32, [32]).  Keys (one random evk shared
    # by every Galois element) and constants are uniform residues made on the device: the cost
    # is data-independent (correctness: tests/test_gpu_apps.py).
    apps_block = None
    if not args.no_apps:
        from paper_conf_isca_jiaodwfcm0z25_b200 import apps as gapps
        gen = torch.Generator(device="cuda")
        gen.manual_seed(seed + 321)
        rnd = lambda *shape: torch.randint(0, 1 << 35, shape, dtype=torch.int64, device="cuda",
                                           generator=gen).view(torch.uint64)
        evk_r = rnd(DNUM, 2, NUM_Q + NUM_P, N)
        f_h, B_h, C_c, H_c = 256, 8, 16, 32
        baby, giant = gapps.conv_rotations(C_c, H_c)
        akeys = {"relin": neo.EvalKey(ctx, evk_r)}
        pool_r, fc_r = gapps.head_rotations(C_c, H_c)
        for r in gapps.helr_rotations(N, f_h) + giant + pool_r:
            akeys.setdefault(gapps.galois(N, r), neo.EvalKey(ctx, evk_r))
        for r in baby + fc_r:
            akeys.setdefault(("h", gapps.galois(N, r)), neo.EvalKey(ctx, evk_r, hoisted_galois=gapps.galois(N, r)))
        del evk_r
        aconsts = {k: rnd(LEVEL + 1, N) for k in gapps.helr_const_names() + gapps.conv_const_names(C_c)
                   + gapps.block_const_names(C_c) + gapps.head_const_names(C_c)}
        aev = gapps.Evaluator(ctx, akeys, aconsts, max_batch=B_h)
        Zc, Wc, Xc = rnd(B_h, 2, LEVEL + 1, N), rnd(1, 2, LEVEL + 1, N), rnd(1, 2, LEVEL + 1, N)

        def timed(fn, reps):
            """(eager ms, graph-replay ms or None); the replay's output is checked equal."""
            out = [None, None]
            for _ in range(2):
                ref = fn()
            torch.cuda.synchronize()
            ref = ref.clone()
            gr, gout = graph_capture(fn)
            if gr is not None:
                gr.replay()
                torch.cuda.synchronize()
                assert _same(gout, ref), "graph replay of the trace differs from the eager run"
            if not agree(gr is not None):
                gr = None
            for i, run in enumerate([fn, gr.replay if gr is not None else None]):
                if run is None:
                    continue
                barrier()
                a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a0.record()
                for _ in range(reps):
                    run()
                a1.record()
                torch.cuda.synchronize()
                tms = a0.elapsed_time(a1) / reps
                if world > 1:
                    t = torch.tensor([tms], dtype=torch.float64, device="cuda")
                    dist.all_reduce(t, op=dist.ReduceOp.MAX)
                    tms = float(t.item())
                out[i] = tms
            return out
        hms_e, hms_g = timed(lambda: gapps.helr_iteration(aev, f_h, Zc, Wc, LEVEL)[0], 3)
        cms_e, cms_g = timed(lambda: gapps.conv_layer(aev, C_c, H_c, Xc, LEVEL)[0], 3)
        bms_e, bms_g = timed(lambda: gapps.head(aev, C_c, H_c, *gapps.basic_block(aev, C_c, H_c, Xc, LEVEL))[0], 3)
        hms = hms_g if hms_g is not None else hms_e
        cms = cms_g if cms_g is not None else cms_e
        bms = bms_g if bms_g is not None else bms_e
        lf, lr = int(math.log2(f_h)), int(math.log2(N // 2 // f_h))
        apps_block = {
            "helr_iteration": {
                "config": "Set-B, l=35, 1024 samples x 256 features (196 padded) = 8 ciphertexts of 128 x 256 slots",
                "ms_per_iteration": round(hms, 3), "value": world / (hms / 1e3), "unit": "iterations/s",
                "graph": hms_g is not None, "ms_eager": round(hms_e, 3),
                "ops": {"hmult": 4 * B_h, "hrot": (2 * lf + lr) * B_h, "pmult": 3 * B_h + 1, "rescale": 7 * B_h + 1},
                "paper_context": "Table 5 (L534-549): Neo 0.22 s per HELR iteration, Set-C, A100 (context only)"},
            "resnet20_conv_layer": {
                "config": "Set-B, l=35, 16 channels x 32 x 32, 3x3 conv (8 hoisted + 15 giant-step HROT, 144 fused PMULT terms) + bias + degree-4 ReLU",
                "ms_per_layer": round(cms, 3), "value": world / (cms / 1e3), "unit": "layers/s",
                "graph": cms_g is not None, "ms_eager": round(cms_e, 3),
                "ops": {"hrot": len(baby) + len(giant), "hmult": 2, "pmult_terms": 9 * C_c + 3},
                "paper_context": "Table 5: Neo 12.03 s for all of ResNet-20 incl. bootstrapping, Set-C, A100 (context only)"},
            "resnet20_block_and_head": {
                "config": "Set-B, l=35 -> 25: a stride-1 basic block (conv, ReLU, conv, + shortcut, ReLU) at 16 x 32 x 32, "
                          "then global average pooling (10 rotate-and-sum HROT) and a 16 -> 16 fully connected layer",
                "ms": round(bms, 3), "value": world / (bms / 1e3), "unit": "block+head/s", "graph": bms_g is not None,
                "ms_eager": round(bms_e, 3),
                "ops": {"hrot": 2 * (len(baby) + len(giant)) + len(pool_r) + len(fc_r), "hmult": 4,
                        "pmult_terms": 2 * (9 * C_c + 3) + 1 + C_c}},
            "timing": "CUDA events around 3 graph replays (headline) and 3 eager runs after warm-ups, max over "
                      "ranks; replay output checked equal to the eager run; synthetic keys/constants"}
        del akeys, aconsts, aev, Zc, Wc, Xc
        torch.cuda.empty_cache()

    # end-to-end through the public API with pinned host buffers: every step copies its three
    # input ciphertexts host->device and both results device->host.  Copies run on their own
    # streams, double-buffered, so the H2D of step k+1 and the D2H of step k-1 overlap the
    # compute of step k (PCIe is full duplex).
    e2e = None
    e2e_u64 = None
    e2e_wire = None
    if not args.no_e2e:
        # two variants through the public API: (u64) residues copied as 8-byte words; (wire) the
        # library's 36-bit wire format (neo_wire_pack/unpack: 4.5 bytes per residue), unpacked
        # on the device before the step and the results packed after it -- inside the region.
        pinned = [[torch.from_numpy(x).pin_memory() for x in slot] for slot in host_in]
        sets = [[torch.empty_like(x) for x in dev_in[0]] for _ in range(2)]
        outs = [new_outs() for _ in range(2)]
        host_out = [(torch.empty(o[1].shape, dtype=torch.uint64).pin_memory(),
                     torch.empty(o[2].shape, dtype=torch.uint64).pin_memory()) for o in outs]
        n_in = [x.numel() for x in dev_in[0]]
        wb_in = [neo.neo_wire_bytes(n) for n in n_in]
        n_out = [outs[0][1].numel(), outs[0][2].numel()]
        wb_out = [neo.neo_wire_bytes(n) for n in n_out]
        off_in = [sum(wb_in[:i]) for i in range(3)]
        off_out = [0, wb_out[0]]
        pinned_w = []
        for slot in dev_in:
            wdev = torch.empty(sum(wb_in), dtype=torch.uint8, device="cuda")
            for i, x in enumerate(slot):
                neo.neo_wire_pack(ctx, x, wdev[off_in[i]:off_in[i] + wb_in[i]])
            pinned_w.append(wdev.cpu().pin_memory())
        wire_in = [torch.empty(sum(wb_in), dtype=torch.uint8, device="cuda") for _ in range(2)]
        wire_out = [torch.empty(sum(wb_out), dtype=torch.uint8, device="cuda") for _ in range(2)]
        host_wout = [torch.empty(sum(wb_out), dtype=torch.uint8).pin_memory() for _ in range(2)]
        h2d_st, d2h_st = torch.cuda.Stream(), torch.cuda.Stream()
        ev_in = [torch.cuda.Event() for _ in range(2)]
        ev_comp = [torch.cuda.Event() for _ in range(2)]
        ev_out = [torch.cuda.Event() for _ in range(2)]
        k_e2e = max(3, min(args.steps, 200))

        def e2e_run(K, wire):
            main = torch.cuda.current_stream()
            for k in range(K):
                s_ = k % 2
                with torch.cuda.stream(h2d_st):
                    if k >= 2:
                        h2d_st.wait_event(ev_comp[s_])
                    if wire:
                        wire_in[s_].copy_(pinned_w[k % SLOTS], non_blocking=True)
                    else:
                        for i in range(3):
                            sets[s_][i].copy_(pinned[k % SLOTS][i], non_blocking=True)
                    ev_in[s_].record(h2d_st)
                main.wait_event(ev_in[s_])
                if k >= 2:
                    main.wait_event(ev_out[s_])
                if wire:
                    for i in range(3):
                        neo.neo_wire_unpack(ctx, wire_in[s_][off_in[i]:off_in[i] + wb_in[i]], sets[s_][i])
                step(0, *sets[s_], outs=outs[s_])
                if wire:
                    for j in range(2):
                        neo.neo_wire_pack(ctx, outs[s_][1 + j], wire_out[s_][off_out[j]:off_out[j] + wb_out[j]])
                ev_comp[s_].record(main)
                with torch.cuda.stream(d2h_st):
                    d2h_st.wait_event(ev_comp[s_])
                    if wire:
                        host_wout[s_].copy_(wire_out[s_], non_blocking=True)
                    else:
                        host_out[s_][0].copy_(outs[s_][1], non_blocking=True)
                        host_out[s_][1].copy_(outs[s_][2], non_blocking=True)
                    ev_out[s_].record(d2h_st)
            for s_ in range(2):
                main.wait_event(ev_out[s_])

        def e2e_time(wire):
            e2e_run(2, wire)
            torch.cuda.synchronize()
            barrier()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            e2e_run(k_e2e, wire)
            e1.record()
            torch.cuda.synchronize()
            ems = e0.elapsed_time(e1)
            if world > 1:
                t = torch.tensor([ems], dtype=torch.float64, device="cuda")
                dist.all_reduce(t, op=dist.ReduceOp.MAX)
                ems = float(t.item())
            return ems

        ems = e2e_time(False)
        e2e_u64 = {"value": 2 * B * world / (ems / k_e2e / 1e3), "unit": UNIT,
                   "h2d_bytes_per_step": sum(n * 8 for n in n_in), "d2h_bytes_per_step": sum(n * 8 for n in n_out),
                   "steps": k_e2e, "ms_per_step": ems / k_e2e, "format": "u64 residues (8 bytes each)"}
        wms = e2e_time(True)
        # the wire round trip is lossless: the last step's packed results unpack to its outputs
        chk = torch.empty_like(outs[(k_e2e - 1) % 2][2])
        neo.neo_wire_unpack(ctx, host_wout[(k_e2e - 1) % 2].cuda()[off_out[1]:], chk)
        torch.cuda.synchronize()
        assert torch.equal(chk.view(torch.int64), outs[(k_e2e - 1) % 2][2].view(torch.int64)), "wire round trip"
        # the PCIe ceiling of this e2e: raw pinned copies of 64 MB, both directions at once
        # (tools/pcie_bw.py): the step's H2D bytes at the per-direction duplex rate
        nb_ = 64 << 20
        hb_i, hb_o = torch.empty(nb_, dtype=torch.uint8).pin_memory(), torch.empty(nb_, dtype=torch.uint8).pin_memory()
        db_i, db_o = torch.empty(nb_, dtype=torch.uint8, device="cuda"), torch.empty(nb_, dtype=torch.uint8, device="cuda")

        def duplex():
            with torch.cuda.stream(h2d_st):
                db_i.copy_(hb_i, non_blocking=True)
            with torch.cuda.stream(d2h_st):
                hb_o.copy_(db_o, non_blocking=True)
            torch.cuda.current_stream().wait_stream(h2d_st)
            torch.cuda.current_stream().wait_stream(d2h_st)
        duplex()
        torch.cuda.synchronize()
        p0, p1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        p0.record()
        for _ in range(10):
            duplex()
        p1.record()
        torch.cuda.synchronize()
        per_dir = nb_ / (p0.elapsed_time(p1) / 10 / 1e3) / 1e9            # GB/s per direction
        bound_ms = max(sum(wb_in), sum(wb_out)) / (per_dir * 1e9) * 1e3
        del hb_i, hb_o, db_i, db_o
        bound_u64 = max(sum(n * 8 for n in n_in), sum(n * 8 for n in n_out)) / (per_dir * 1e9) * 1e3
        # headline e2e: the caller's u64 host buffers (the ABI's own layout) copied in and out every
        # step, nothing prepared outside the region
        e2e = dict(e2e_u64, pcie={"duplex_GBps_per_direction": round(per_dir, 1),
                                  "bound_ms_per_step": round(bound_u64, 4),
                                  "frac_of_bound": round(bound_u64 / (ems / k_e2e), 3),
                                  "note": "raw pinned 64 MB copies in both directions at once; the step's larger "
                                          "direction (H2D, 113 MB) at that rate is the e2e ceiling"},
                   overlap="H2D / compute / D2H on separate streams, double-buffered")
        e2e_wire = {"value": 2 * B * world / (wms / k_e2e / 1e3), "unit": UNIT,
                    "h2d_bytes_per_step": sum(wb_in), "d2h_bytes_per_step": sum(wb_out),
                    "steps": k_e2e, "ms_per_step": wms / k_e2e,
                    "bound_ms_per_step": round(bound_ms, 4), "frac_of_bound": round(bound_ms / (wms / k_e2e), 3),
                    "format": "host buffers already in the library's 36-bit wire format (4.5 bytes per residue; "
                              "packed once before the region, as a caller storing ciphertexts in that format "
                              "would); unpack / pack on the device inside the region",
                    "note": "secondary: not the headline e2e because the packing of the inputs is outside the region"}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        d0 = host_in[0][2][0, 1]                                  # c1 of one ciphertext: [36][N]
        rate, reps, el, cores = oracle_keyswitch_rate(d0, rot_np)
        cpu = {"value": rate, "unit": UNIT, "cores": cores, "kind": "oracle",
               "sample": f"{reps} Set-B key-switch(es) (l=35, B=1) by the CPU oracle in {el:.1f} s",
               "host": host_cpu_info(), "tiny_definitional": oracle_tiny_def_timing()}

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "weak",
                "vs_baseline": None, "dtype": "u64", "data": "synthetic (uniform residues, random keys)",
                "config": dict(workload_config(B, world),
                               hmult_rescale="one neo_hmult_rescale call" if args.fused_rescale
                               else "neo_hmult then neo_rescale",
                               steps_per_graph=CH,
                               chains=("each stream runs its chain of HMULT+Rescale / HROTATE steps back to "
                                       f"back, joined every {CH} steps (one CUDA graph)") if CH > 1
                               else "streams joined after every step"),
                "roofline": {"bound": "hbm", "kernel": dom, "achieved": achieved, "peak": peak,
                             "peak_source": peak_src, "unit": "GB/s",
                             "frac": achieved / peak if achieved else None, "traffic": traffic,
                             "launches_per_step": n_launch_dom, "algo_bytes_per_step": bm[dom],
                             "bytes_rule": "SURVEY §8(d): one read + one write per limb an operation transforms, "
                                           "plus fused-epilogue operands (bench.bytes_model)",
                             "ntt_impl": ntt_impl, "ntt_transforms_per_step": n_transforms, "alt": alt},
                "step_roofline": {"algo_bytes_per_step": sum(bm.values()),
                                  "achieved": sum(bm.values()) / (ms_step / 1e3) / 1e9,
                                  "peak": peak, "unit": "GB/s",
                                  "frac": sum(bm.values()) / (ms_step / 1e3) / 1e9 / peak,
                                  "note": "whole step (all kernels, 2 streams) against HBM, per GPU"},
                "cpu_baseline": cpu, "e2e": e2e, "e2e_wire": e2e_wire, "gpu_launches": gpu_launches, "hoisted_rotations": hoisted, "latency": latency,
                "limb_sharded_keyswitch": sharded_ks, "limb_sharded_keyswitch_native": sharded_native,
                "batch_hrot": batch_block, "klss_vs_hybrid_setc": klss_block, "bootstrap": boot_block, "apps": apps_block,
                "clocks": clk.summary(), "graph": bool(args.graph), "streams": args.streams,
                "single_stream_profiled_ms_per_step": ms_step_1s, "breakdown": breakdown}
        emit(line)
    if world > 1:
        dist.destroy_process_group()


_JSON_OUT = None


def emit(line: dict):
    """The one JSON line, on the process's original stdout (everything else goes to stderr)."""
    out = _JSON_OUT if _JSON_OUT is not None else sys.stdout
    out.write(json.dumps(line) + "\n")
    out.flush()


def main():
    global _JSON_OUT
    # keep stdout to the JSON line alone: libraries (NCCL's version banner, ...) print to fd 1
    sys.stdout.flush()
    _JSON_OUT = os.fdopen(os.dup(1), "w")
    os.dup2(2, 1)
    args = parse()
    if args.impl == "reference":
        run_reference(args)
    else:
        run_neo(args)


if __name__ == "__main__":
    main()
