#!/usr/bin/env python
"""bench.py — FLBooster hot path on B200: Paillier ops/s at 2048-bit keys (BASELINE.json metric).

Workload (BASELINE.json configs[1], "C2"): Homo-LR gradient aggregation.  Per rank, 8 clients
each hold a 1,048,576-element float32 gradient (synthetic, N(0, 0.05^2) clipped, 1 % at +-1).
One step is one pass of the whole hot path:
    pack (Eq. 6–9, w = 32, S = 63)  ->  encrypt 8 x 16,645 plaintexts (Eq. 3, Philox r)
    ->  segmented product over clients (Eq. 5)  [N > 1: all_to_all + N-way product]
    ->  CRT decrypt (Eq. 4)  ->  unpack + dequantise (L297, cnt = clients)
metric value = (encryptions + decryptions + homomorphic additions) per second over all ranks.

  python bench.py [--gpus N --steps K --warmup W]          # this library (CUDA)
  python bench.py --impl reference                         # the CPU oracle on the host cores
Multi-GPU: python -m torch.distributed.run --nproc-per-node N bench.py --gpus N ... (weak
scaling: every rank hosts 8 clients of an 8N-client federation; rows are reduce-scattered).
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

CLIENTS = 8            # clients per rank (C2: "summed over 8 clients")
N_VALUES = 1 << 20     # gradient length (Avazu-sized)
KEY_BITS = 2048
KEY_SEED = 0xF1B0 + 2048
ALPHA = 1.0
SLOT_BITS = 32         # slots a multiple of 32 bits
METRIC = "Paillier encrypt/decrypt/hom-add ops/sec at 2048-bit key, 1/2/4/8 B200"
HBM_GBS = 6549.1  # MEASURED_PEAKS.json hbm_gbs (copy bandwidth), re-read below when the file is present
try:
    with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as _f:
        HBM_GBS = float(__import__("json").load(_f).get("hbm_gbs", HBM_GBS))
except (OSError, ValueError):
    pass
UNIT = "ops/s"
PEAK_LP_PER_CLK_SM = 32  # NOMINAL: IMAD.WIDE.U32(.X) at half rate on the FMA-heavy pipe (B300 guide: IMAD rt=2/SMSP)
# measured ceilings of carry-chained IMAD.WIDE.U32.X sequences (tools/chain_lat.cu, profiles/r02_chain_lat.jsonl;
# tools/imad_peak.cu, profiles/r01_imad_peak.jsonl): context for the nominal peak, not the denominator
MEASURED_LP_PER_CLK_SM = {"chain_lat 2-chain, 16-64 warps/SM": 22.3, "imad_peak 1-chain, 64 warps/SM": 28.0}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["flb", "reference"], default="flb")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--cpu-sample-seconds", type=float, default=20.0)
    ap.add_argument("--workload", choices=["c2", "c1", "c3", "c4", "c5"], default="c2",
                    help="BASELINE.json configs: c2 (default, the headline) or c1/c3/c4/c5 (single GPU)")
    ap.add_argument("--c5-ops", type=int, default=0, help="c5 batch per key size (default: 1M / 256K)")
    ap.add_argument("--encrypt", choices=["keyholder", "public"], default="keyholder",
                    help="C2 clients hold the key pair (they decrypt the aggregate, Fig. 2), so they may "
                         "encrypt by CRT; 'public' uses the public-key-only kernel")
    return ap.parse_args()


def codec_params(world: int):
    participants = CLIENTS * world
    pad = max(1, math.ceil(math.log2(participants)))  # b = ceil(log2 p)
    return ALPHA, SLOT_BITS - pad, pad


# ----------------------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region (B200_PROFILING.md)."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device_index: int):
        self.dev = device_index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.dev), "--query-gpu=" + self.FIELDS, "--format=csv,noheader,nounits",
                 "-lms", "200"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except (OSError, FileNotFoundError):
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        sm, mx, reasons, power = [], [], set(), []
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 9:
                continue
            try:
                sm.append(float(parts[1]))
                mx.append(float(parts[2]))
                power.append(float(parts[3]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        loaded = [s for s in sm if s > 500] or sm
        return {"sm_mhz": statistics.median(loaded) if loaded else None,
                "sm_max_mhz": max(mx) if mx else None,
                "power_w_max": max(power) if power else None,
                "samples": len(sm), "reasons": sorted(reasons)}


# ----------------------------------------------------------------------------- CPU oracle timing
def _oracle_enc(args):
    from oracle import paillier, philox
    n, m, seed, idx, ptw = args
    return paillier.encrypt(n, m, philox.draw_r(n, seed, idx, ptw))


def _oracle_dec(args):
    from oracle import paillier
    p, q, c = args
    return paillier.decrypt(p, q, c)


def oracle_rates(sample_seconds: float, cores: int):
    """Time the oracle as it stands on the host cores (multiprocessing over a bounded sample).
    Returns per-op wall seconds (with `cores` workers) and a description of the sample."""
    import multiprocessing as mp
    import random
    import numpy as np
    import synthetic
    from oracle import codec, paillier
    p, q = paillier.keygen(KEY_BITS, KEY_SEED)  # the oracle's own key of the same size
    n = p * q
    n2 = n * n
    ptw = KEY_BITS // 32
    rng = random.Random(1)
    # size the sample from a single-op calibration so the whole leg takes ~sample_seconds
    t0 = time.perf_counter()
    _oracle_enc((n, rng.randrange(n), 7, 0, ptw))
    t_enc1 = time.perf_counter() - t0
    budget = sample_seconds * cores
    n_enc = max(cores, int(0.7 * budget / t_enc1) // cores * cores)
    n_dec = max(cores, n_enc // 2)
    ms = [rng.randrange(n) for _ in range(n_enc)]
    ctx = mp.get_context("fork")
    with ctx.Pool(cores) as pool:
        t0 = time.perf_counter()
        cs = pool.map(_oracle_enc, [(n, ms[i], 7, i, ptw) for i in range(n_enc)], chunksize=1)
        t_enc = (time.perf_counter() - t0) / n_enc
        t0 = time.perf_counter()
        pool.map(_oracle_dec, [(p, q, cs[i % n_enc]) for i in range(n_dec)], chunksize=1)
        t_dec = (time.perf_counter() - t0) / n_dec
    # hom-add (single process; microseconds each)
    k = 2000
    t0 = time.perf_counter()
    acc = cs[0]
    for i in range(k):
        acc = paillier.add(n, acc, cs[i % n_enc])
    t_add = (time.perf_counter() - t0) / k / cores  # embarrassingly parallel across cores
    # codec: pack + unpack of a sample of one client's gradient
    x = synthetic.c2_gradient(0)[: 63 * 64]
    alpha, qb, pb = codec_params(1)
    t0 = time.perf_counter()
    z = codec.pack([float(v) for v in x], alpha, qb, pb, 63)
    codec.unpack(z, len(x), alpha, qb, pb, 63, CLIENTS)
    t_codec_value = (time.perf_counter() - t0) / len(x) / cores
    sample = ("oracle (pure-Python ints): %d encryptions + %d CRT-free decryptions on %d processes, "
              "%d hom-adds, pack+unpack of %d values; extrapolated to the C2 step mix"
              % (n_enc, n_dec, cores, k, len(x)))
    return {"t_enc": t_enc, "t_dec": t_dec, "t_add": t_add, "t_codec_value": t_codec_value, "sample": sample}


def c2_step_ops(rows: int, world: int):
    enc = CLIENTS * rows * world
    adds = (CLIENTS - 1) * rows * world + (world - 1) * rows
    dec = rows
    return enc, dec, adds


def oracle_value(r, rows: int):
    enc, dec, adds = c2_step_ops(rows, 1)
    step = enc * r["t_enc"] + dec * r["t_dec"] + adds * r["t_add"] + (CLIENTS + 1) * N_VALUES * r["t_codec_value"]
    return (enc + dec + adds) / step, step


def cpu_cores():
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:
        return os.cpu_count() or 1


# ----------------------------------------------------------------------------- reference arm
def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    from oracle import codec
    cores = cpu_cores()
    rows = codec.num_plaintexts(N_VALUES, 63)
    per = max(3.0, 60.0 / max(1, args.steps + args.warmup))
    vals = []
    for s in range(args.warmup + args.steps):
        r = oracle_rates(per, cores)
        v, step_s = oracle_value(r, rows)
        if s >= args.warmup:
            vals.append((v, step_s, r["sample"]))
    v = statistics.median([x[0] for x in vals])
    line = {
        "impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * statistics.median([x[1] for x in vals]),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32-limb bigint (+f64 codec)",
        "data": "synthetic",
        "config": {"workload": "C2 Homo-LR aggregation, 2048-bit key, 8 clients x 1,048,576 values",
                   "note": "CPU oracle: each step times a bounded sample (about %.0f s of CPU work) and "
                           "extrapolates to the C2 step; ms_per_step is that extrapolated step time, not the "
                           "wall clock of this run" % per},
        "ms_per_step_extrapolated": True,
        "cpu_baseline": {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": vals[-1][2]},
        "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ----------------------------------------------------------------------------- CUDA arm
def run_flb(args):
    import numpy as np
    import torch
    import torch.distributed as dist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    backend = os.environ.get("FLB_DIST_BACKEND", "nccl")  # gloo: multi-rank logic check on one GPU
    if world > 1:
        torch.cuda.set_device(local % torch.cuda.device_count())
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    else:
        torch.cuda.set_device(0)
    dev = torch.device("cuda", torch.cuda.current_device())

    import paper_conf_icde_zeng0fcpcwg23_b200 as flb
    from paper_conf_icde_zeng0fcpcwg23_b200 import dist as fdist
    import synthetic

    pub, priv = flb.keygen(KEY_BITS, KEY_SEED)  # product keygen (C++ host), same key on every rank
    alpha, qbits, pad = codec_params(world)
    S = pub.slot_capacity(SLOT_BITS)            # 63 at 2048 bits (reading c16)
    cd = flb.Codec(alpha, qbits, pad, S)
    rows = cd.num_plaintexts(N_VALUES)          # 16,645
    rows_p = fdist.padded_rows(rows, world)
    rpr = rows_p // world
    ptw, ctw = pub.pt_words, pub.ct_words

    # inputs resident in HBM before timing
    grads_host = [torch.from_numpy(synthetic.c2_gradient(CLIENTS * rank + c)) for c in range(CLIENTS)]
    grads = [g.to(dev) for g in grads_host]
    offs, idx = fdist.client_segments(CLIENTS, rows, rows_p, device=dev)
    pt = torch.empty((CLIENTS * rows, ptw), dtype=torch.int32, device=dev)
    ct = torch.empty((CLIENTS * rows, ctw), dtype=torch.int32, device=dev)
    part = torch.empty((rows_p, ctw), dtype=torch.int32, device=dev)
    recv = torch.empty_like(part)
    fin = torch.empty((rpr, ctw), dtype=torch.int32, device=dev)
    dec = torch.empty((rpr, ptw), dtype=torch.int32, device=dev)
    r0, r1 = fdist.rank_rows(rows, world, rank)
    my_values = max(0, min(N_VALUES, r1 * S) - r0 * S)
    out = torch.empty((max(my_values, 1),), dtype=torch.float32, device=dev)
    foffs, fidx = fdist.finish_segments(world, rpr, device=dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)

    def reduce_cb(buf, o, i, L):
        return flb.reduce_segments(pub, buf, o, idx=i, max_segment_len=L, out=fin)

    ev = {}

    def mark(name):
        e = torch.cuda.Event(enable_timing=True)
        e.record()
        ev.setdefault(name, []).append(e)

    def step(s, gsrc=None):
        seed = 0xC2000000 + s
        mark("t0")
        for c in range(CLIENTS):
            flb.pack(pub, cd, grads[c] if gsrc is None else gsrc[c], out=pt[c * rows:(c + 1) * rows])
        mark("t_pack")
        if args.encrypt == "keyholder":
            flb.encrypt_crt(priv, pt, seed=seed, ctr0=rank * CLIENTS * rows, out=ct)
        else:
            flb.encrypt(pub, pt, seed=seed, ctr0=rank * CLIENTS * rows, out=ct)
        mark("t_enc")
        flb.reduce_segments(pub, ct, offs, idx=idx, max_segment_len=CLIENTS, out=part)
        mark("t_red")
        if world > 1:
            fdist.exchange_and_finish(part, None, reduce_cb, world, recv=recv)
            agg = fin
        else:
            agg = part
        mark("t_xchg")
        flb.decrypt(priv, agg[: (r1 - r0) if world > 1 else rows], out=dec[: (r1 - r0) if world > 1 else rows])
        mark("t_dec")
        if my_values:
            flb.unpack(pub, cd, dec, my_values, summands=CLIENTS * world, out=out[:my_values])
        mark("t_unpack")

    ops_enc, ops_dec, ops_add = c2_step_ops(rows, world)
    total_ops = ops_enc + ops_dec + ops_add

    for s in range(args.warmup):
        step(s)
    torch.cuda.synchronize()
    ev.clear()

    clocks = ClockSampler(torch.cuda.current_device())
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks.start()
    step_ms = []
    for s in range(args.steps):
        flush.zero_()
        step(1000 + s)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clk = clocks.stop()

    names = ["t0", "t_pack", "t_enc", "t_red", "t_xchg", "t_dec", "t_unpack"]
    phase = {n: 0.0 for n in names[1:]}
    for s in range(args.steps):
        step_ms.append(ev["t0"][s].elapsed_time(ev["t_unpack"][s]))
        for a, b in zip(names[:-1], names[1:]):
            phase[b] += ev[a][s].elapsed_time(ev[b][s]) / args.steps
    ms = sum(step_ms) / len(step_ms)
    if world > 1:
        t = torch.tensor([ms] + [phase[n] for n in names[1:]], dtype=torch.float64,
                         device=dev if backend == "nccl" else "cpu")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t[0])
        for i, n in enumerate(names[1:]):
            phase[n] = float(t[i + 1])
    value = total_ops / (ms * 1e-3)

    # the other encryption path, timed once on the same batch (reported, not part of the step)
    other = "public" if args.encrypt == "keyholder" else "keyholder"

    def other_enc():
        if other == "public":
            flb.encrypt(pub, pt, seed=7, out=ct)
        else:
            flb.encrypt_crt(priv, pt, seed=7, out=ct)
    other_enc()  # warm-up
    other_ms = []
    for _ in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        other_enc()
        e1.record()
        torch.cuda.synchronize()
        other_ms.append(e0.elapsed_time(e1))
    other_rate = ops_enc / world / (statistics.median(other_ms) * 1e-3)

    # roofline of the dominant kernel (encrypt): algorithmic limb products / its event time
    tc_on = os.environ.get("FLB_TC", "1") != "0"
    dag_on = os.environ.get("FLB_TC_DAG", "1") != "0" and KEY_BITS == 2048
    enc_tc = dec_tc = None
    if tc_on:
        try:
            enc_tc = flb.op_cost(priv, "encrypt_crt_tc")
            dec_tc = flb.op_cost(priv, "decrypt_tc")
            enc_macs = flb.op_cost(priv, "encrypt_crt_tc_macs")[1]
        except flb.FlbError:
            enc_tc = dec_tc = None
    if args.encrypt == "keyholder":
        enc_mm, enc_lp = flb.op_cost(priv, "encrypt_crt")
        if enc_tc and dag_on:
            enc_kernel = ("k_tc_exp_dag<32,64> (both key-holder stages in one launch, stage-2 tiles wait on their "
                          "stage-1 tile; Montgomery reduction as u8 tcgen05 MMAs, t = a b on the IMAD pipe)")
        elif enc_tc:
            enc_kernel = ("k_tc_exp<32> + k_tc_exp<64> (two-stage key-holder encryption; Montgomery reduction as "
                          "u8 tcgen05 MMAs, t = a b on the IMAD pipe)")
        else:
            enc_kernel = "k_crt_pre<16,2> + k_encrypt_crt2<16,4> (two-stage key-holder encryption)"
    else:
        enc_mm, enc_lp = flb.op_cost(pub, "encrypt")
        enc_tc = None
        if tc_on:
            try:  # public-key encryption in the n^2 frame on the tensor cores (k_tc_exp<128> at 2048 bits)
                enc_tc = flb.op_cost(pub, "encrypt_tc")
                enc_macs = flb.op_cost(pub, "encrypt_tc_macs")[1]
            except flb.FlbError:
                enc_tc = None
        enc_kernel = ("k_tc_exp<%d> (public-key encryption (1 + m n) r^n mod n^2 in the n^2 frame; Montgomery "
                      "reduction as u8 tcgen05 MMAs, t = a b on the IMAD pipe)" % ctw) if enc_tc else "k_encrypt<16,8>"
    dec_mm, dec_lp = flb.op_cost(priv, "decrypt")
    enc_units = CLIENTS * rows
    sm_mhz_max = clk.get("sm_max_mhz") or 1965.0
    peak = 148 * PEAK_LP_PER_CLK_SM * sm_mhz_max * 1e6 / 1e12
    # u8 MMA peak: tools/tc_i8_probe.cu measured 7.26K MAC/clk/SM (kind::i8, M=128 N=256)
    mma_peak = 148 * 7260 * sm_mhz_max * 1e6 / 1e12
    if enc_tc:
        # IMAD-pipe work the tensor-core kernels actually issue: S^2 per Montgomery product
        imad_lp = enc_tc[1]
        achieved = imad_lp * enc_units / (phase["t_enc"] * 1e-3) / 1e12
        per_unit = {"mont_muls": enc_tc[0], "imad_limb_products": imad_lp, "u8_macs": enc_macs,
                    "cios_equivalent_limb_products": enc_lp}
        tensor = {"achieved": enc_macs * enc_units / (phase["t_enc"] * 1e-3) / 1e12, "peak": mma_peak,
                  "unit": "T u8 MAC/s (tcgen05.mma kind::i8)",
                  "peak_basis": "148 SM x 7.26K MAC/clk/SM (tools/tc_i8_probe.cu) x %.0f MHz" % sm_mhz_max}
        tensor["frac"] = tensor["achieved"] / mma_peak
        cios_eq = enc_lp * enc_units / (phase["t_enc"] * 1e-3) / 1e12
    else:
        achieved = enc_lp * enc_units / (phase["t_enc"] * 1e-3) / 1e12
        per_unit = {"mont_muls": enc_mm, "limb_products": enc_lp}
        tensor = None
        cios_eq = achieved
    dec_roof = None
    if dec_tc:
        dec_roof = {"kernel": "k_tc_exp<64> + k_dec_finish<16,4>", "mont_muls_tc": dec_tc[0],
                    "imad_limb_products": dec_tc[1],
                    "imad_achieved": dec_tc[1] * rows / (phase["t_dec"] * 1e-3) / 1e12,
                    "frac": dec_tc[1] * rows / (phase["t_dec"] * 1e-3) / 1e12 / peak}
    # the HBM-bound steps: bytes each moves per step / its event time (pack: float32 in, plaintext limbs
    # out; unpack: plaintext limbs in, float32 out; reduce: CLIENTS ciphertexts in per row, one out)
    add_lp = flb.op_cost(pub, "add")[1] // 2  # one Montgomery product (CIOS limb products) per reduce input
    hbm = {
        "pack": {"bytes": 4 * N_VALUES * CLIENTS + 4 * CLIENTS * rows * ptw, "ms": phase["t_pack"]},
        "unpack": {"bytes": (r1 - r0 if world > 1 else rows) * ptw * 4 + 4 * my_values, "ms": phase["t_unpack"]},
        "reduce": {"bytes": (CLIENTS + 1) * rows_p * ctw * 4 + 8 * (rows_p + 1 + CLIENTS * rows), "ms": phase["t_red"]},
    }
    for k, d in hbm.items():
        d["GB_per_s"] = d["bytes"] / (d["ms"] * 1e-3) / 1e9 if d["ms"] > 0 else None
        d["frac_of_measured_hbm"] = d["GB_per_s"] / HBM_GBS if d["GB_per_s"] else None
    red_units = CLIENTS * rows
    op_fracs = {
        "encrypt (IMAD limb products of the dominant kernel)": achieved / peak,
        "decrypt": dec_roof["frac"] if dec_roof else None,
        "reduce (hom-add products, k_reduce CIOS)": add_lp * red_units / (phase["t_red"] * 1e-3) / 1e12 / peak,
    }
    traffic = None
    # DRAM bytes per launch of the dominant kernel from the round's ncu --set full capture
    # (tools/traffic_from_ncu.py)
    if args.encrypt == "public":
        tp = "r02_encrypt_pub_tc_traffic.json" if tc_on else "encrypt_traffic.json"
    else:
        tp = "r02_encrypt_tc_traffic.json" if enc_tc else "encrypt_crt_traffic.json"
    tp = os.path.join(ROOT, "profiles", tp)
    if os.path.exists(tp):
        try:
            with open(tp) as f:
                traffic = json.load(f).get("dram_bytes_per_launch")
        except (OSError, ValueError):
            traffic = None

    # e2e: the C-ABI host-buffer pipeline (flb_pack_encrypt_host / flb_reduce_segments_host /
    # flb_decrypt_unpack_host, PAPER Fig. 4): host gradients in, host floats out, every H2D/D2H copy
    # inside the timed region; the cross-rank exchange (N > 1) runs on device buffers.
    e2e = None
    if not args.no_e2e:
        import numpy as np

        def pinned(shape, dtype):
            # page-locked host buffers (the host pipeline DMAs straight from / into them)
            t = torch.empty(shape, dtype=torch.int32 if dtype == np.uint32 else torch.float32, pin_memory=True)
            return t.numpy().view(dtype)

        grads_np = []
        for g in grads_host:
            gp = pinned(tuple(g.shape), np.float32)
            gp[...] = g.numpy()
            grads_np.append(gp)
        offs_np, idx_np = offs.cpu().numpy(), idx.cpu().numpy()
        cts_h = pinned((CLIENTS * rows, ctw), np.uint32)
        part_out = pinned((len(offs_np) - 1, ctw), np.uint32)
        vals_out = pinned((max(my_values, 1),), np.float32)
        kh = priv if args.encrypt == "keyholder" else None
        h2d = d2h = 0

        def e2e_step(s):
            nonlocal h2d, d2h
            h2d = d2h = 0
            flb.pack_encrypt_host_multi(pub, cd, grads_np, seed=3000 + s, ctr0=rank * CLIENTS * rows, priv=kh,
                                        out=cts_h)
            h2d += sum(g.nbytes for g in grads_np)
            d2h += cts_h.nbytes
            part_h = flb.reduce_segments_host(pub, cts_h, offs_np, idx_np, max_segment_len=CLIENTS, out=part_out)
            h2d += cts_h.nbytes + offs_np.nbytes + idx_np.nbytes
            d2h += part_h.nbytes
            if world > 1:
                part_d = torch.from_numpy(part_h.view(np.int32)).to(dev)
                fdist.exchange_and_finish(part_d, None, reduce_cb, world, recv=recv)
                fin_h = fin[: r1 - r0].cpu().numpy().view(np.uint32)
                h2d += part_h.nbytes
                d2h += fin_h.nbytes
            else:
                fin_h = part_h[:rows]
            if my_values:
                flb.decrypt_unpack_host(priv, cd, fin_h, my_values, summands=CLIENTS * world, out=vals_out[:my_values])
                h2d += fin_h.nbytes
                d2h += my_values * 4

        e2e_step(0)  # warm-up (pinned staging allocation)
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for s in range(args.steps):
            e2e_step(1 + s)
        torch.cuda.synchronize()
        e_ms = (time.perf_counter() - t0) * 1e3 / args.steps
        hb = [float(e_ms), float(h2d), float(d2h)]
        if world > 1:
            t = torch.tensor(hb, dtype=torch.float64, device=dev if backend == "nccl" else "cpu")
            dist.all_reduce(t, op=dist.ReduceOp.SUM)
            tm = torch.tensor([e_ms], dtype=torch.float64, device=dev if backend == "nccl" else "cpu")
            dist.all_reduce(tm, op=dist.ReduceOp.MAX)
            e_ms, h2d, d2h = float(tm[0]), float(t[1]), float(t[2])
        e2e = {"value": total_ops / (e_ms * 1e-3), "unit": UNIT, "h2d_bytes_per_step": int(h2d),
               "d2h_bytes_per_step": int(d2h), "ms_per_step": e_ms,
               "path": "C-ABI host-buffer pipeline over page-locked host arrays: flb_pack_encrypt_host_multi (%d clients) -> flb_reduce_segments_host "
                       "-> %sflb_decrypt_unpack_host; host wall clock per step" %
                       (CLIENTS, "NCCL all_to_all + finish -> " if world > 1 else "")}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cores = cpu_cores()
        r = oracle_rates(args.cpu_sample_seconds, cores)
        v, _ = oracle_value(r, rows)
        cpu = {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": r["sample"],
               "per_op_seconds": {"encrypt": r["t_enc"], "decrypt": r["t_dec"], "add": r["t_add"]}}

    # pack per client; encrypt (TC: Philox fill, k_tc_exp_dag (or k_tc_exp<32>, k_tc_exp<64>),
    # k_crt_combine; CIOS: k_crt_pre, k_encrypt_crt2); reduce (plan scan, plan fill, k_reduce);
    # exchange + finish (N > 1); decrypt (TC: k_tc_exp<64>, k_dec_finish; CIOS: k_decrypt); unpack
    enc_launches = ((3 if dag_on else 4) if enc_tc else 2) if args.encrypt == "keyholder" else 1
    launches_per_step = (CLIENTS + enc_launches + 3 + (3 if world > 1 else 0) + (2 if dec_tc else 1)
                         + (1 if my_values else 0))
    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u32-limb bigint (+f64 codec)", "data": "synthetic",
            "config": {"workload": "C2 Homo-LR aggregation: 2048-bit key, %d clients/GPU x 1,048,576 float32 "
                                   "values, packed w=32 S=%d (rho=%d, b=%d), encrypt %d (%s), product over "
                                   "clients, decrypt %d, unpack" % (CLIENTS, S, qbits, pad, CLIENTS * rows * world,
                                                                    args.encrypt, rows),
                       "key_bits": KEY_BITS, "clients_per_gpu": CLIENTS, "values_per_client": N_VALUES,
                       "plaintexts_per_client": rows, "parallelism": "dp%d (shard by ciphertext)" % world,
                       "l2": "flushed between steps (256 MiB memset outside the per-step events)"},
            "breakdown_ms": phase,
            "ops_per_step": {"encrypt": ops_enc, "decrypt": ops_dec, "add": ops_add},
            "op_rates": {"encrypt_per_s": ops_enc / (phase["t_enc"] * 1e-3),
                         "decrypt_per_s": ops_dec / (phase["t_dec"] * 1e-3),
                         "add_per_s": ops_add / ((phase["t_red"] + phase["t_xchg"]) * 1e-3),
                         ("encrypt_public_per_gpu_per_s" if other == "public" else "encrypt_keyholder_per_gpu_per_s"):
                             other_rate},
            "encrypt_mode": args.encrypt,
            "roofline": {"bound": "alu", "kernel": enc_kernel, "achieved": achieved, "peak": peak,
                         "unit": "T limb-products/s (IMAD.WIDE.U32 32x32->64, FMA-heavy pipe)",
                         "frac": achieved / peak, "traffic": traffic, "per_unit": per_unit,
                         "peak_basis": "NOMINAL: 148 SM x 32 IMAD.WIDE/clk/SM x %.0f MHz (guide: IMAD rt=2/SMSP, "
                                       "IMAD.WIDE half rate); nothing in MEASURED_PEAKS.json covers integer work" % sm_mhz_max,
                         "measured_ceilings_lp_per_clk_sm": MEASURED_LP_PER_CLK_SM,
                         "tensor": tensor, "cios_equivalent_achieved": cios_eq,
                         "cios_equivalent_frac": cios_eq / peak},
            "decrypt_cost": {"mont_muls": dec_mm, "limb_products": dec_lp},
            "op_roofline_fracs": op_fracs, "hbm_steps": hbm,
            "decrypt_roofline": dec_roof,
            "clocks": clk, "gpu_launches": launches_per_step * args.steps,
            "e2e": e2e, "cpu_baseline": cpu,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


# ----------------------------------------------------------------------------- other configs
def _timer():
    import torch
    ev = {}

    def mark(name):
        e = torch.cuda.Event(enable_timing=True)
        e.record()
        ev.setdefault(name, []).append(e)
    return ev, mark


def _phases(ev, names, steps):
    out = {n: 0.0 for n in names[1:]}
    total = []
    for s in range(steps):
        total.append(ev[names[0]][s].elapsed_time(ev[names[-1]][s]))
        for a, b in zip(names[:-1], names[1:]):
            out[b] += ev[a][s].elapsed_time(ev[b][s]) / steps
    return sum(total) / len(total), out


def run_other(args):
    """C1, C3, C4, C5 on one GPU (BASELINE.json configs[0], [2], [3], [4])."""
    import numpy as np
    import torch
    import torch.distributed as dist
    import paper_conf_icde_zeng0fcpcwg23_b200 as flb
    import synthetic
    wl = args.workload
    world = int(os.environ.get("WORLD_SIZE", "1")) if wl == "c5" else 1
    rank = int(os.environ.get("RANK", "0")) if world > 1 else 0
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:  # C5 shards by ciphertext (weak scaling); the other configs run on one GPU
        torch.cuda.set_device(local % torch.cuda.device_count())
        backend = os.environ.get("FLB_DIST_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local % torch.cuda.device_count()))
        else:
            dist.init_process_group(backend)
    elif int(os.environ.get("RANK", "0")) != 0:
        return 0  # C1/C3/C4 are single-GPU configs: the other ranks have nothing to do
    else:
        torch.cuda.set_device(0)
    dev = torch.device("cuda", torch.cuda.current_device())
    clk = ClockSampler(torch.cuda.current_device())
    res = {"metric": METRIC, "unit": UNIT, "n_gpus": 1, "steps": args.steps, "warmup": args.warmup,
           "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
           "dtype": "u32-limb bigint (+f64 codec)", "data": "synthetic"}
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    clk.start()

    def run_steps(step, names):
        for s in range(args.warmup):
            step(s)
        torch.cuda.synchronize()
        ev.clear()
        if world > 1:
            dist.barrier()
        for s in range(args.steps):
            flush.zero_()
            step(100 + s)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        return _phases(ev, names, args.steps)

    ev, mark = _timer()
    if wl == "c1":
        pub, priv = flb.keygen(1024, 0xF1B0 + 1024)
        cd = flb.Codec(0.5, 30, 2, 1)
        a, b = synthetic.c1_values()
        ta, tb = torch.from_numpy(a).to(dev), torch.from_numpy(b).to(dev)
        nv = len(a)
        pts = torch.empty((2 * nv, pub.pt_words), dtype=torch.int32, device=dev)
        cts = torch.empty((3 * nv, pub.ct_words), dtype=torch.int32, device=dev)
        dec = torch.empty((3 * nv, pub.pt_words), dtype=torch.int32, device=dev)
        out = torch.empty(3 * nv, dtype=torch.float32, device=dev)

        def step(s):
            mark("t0")
            flb.pack(pub, cd, ta, out=pts[:nv])
            flb.pack(pub, cd, tb, out=pts[nv:])
            mark("pack")
            flb.encrypt(pub, pts, seed=s, out=cts[:2 * nv])
            mark("encrypt")
            flb.add(pub, cts[:nv], cts[nv:2 * nv], out=cts[2 * nv:])
            mark("add")
            flb.decrypt(priv, cts, out=dec)
            mark("decrypt")
            flb.unpack(pub, cd, dec[:2 * nv], 2 * nv, summands=1, out=out[:2 * nv])
            flb.unpack(pub, cd, dec[2 * nv:], nv, summands=2, out=out[2 * nv:])
            mark("unpack")
        names = ["t0", "pack", "encrypt", "add", "decrypt", "unpack"]
        ms, ph = run_steps(step, names)
        ops = 2 * nv + nv + 3 * nv
        res.update(value=ops / (ms * 1e-3), ms_per_step=ms, breakdown_ms=ph,
                   ops_per_step={"encrypt": 2 * nv, "add": nv, "decrypt": 3 * nv},
                   config={"workload": "C1: 1024-bit key, 1,000 fixed-point values a, b ~ U(-0.5, 0.5); "
                                       "encrypt 2,000, pairwise hom-add 1,000, decrypt 3,000 (latency point: "
                                       "cannot fill 148 SMs)", "key_bits": 1024, "codec": "alpha=0.5 rho=30 b=2 S=1"})
    elif wl == "c3":
        pub, priv = flb.keygen(2048, 0xF1B0 + 2048)
        N, F = 1 << 22, 8
        d, x = synthetic.c3_residuals(N, F)
        cd = flb.Codec(1.0, 30, 2, 1)
        td = torch.from_numpy(d).to(dev)
        tx = torch.from_numpy(x.view(np.int32).reshape(N * F, 1)).to(dev)
        pt = torch.empty((N, pub.pt_words), dtype=torch.int32, device=dev)
        ct = torch.empty((N, pub.ct_words), dtype=torch.int32, device=dev)
        ctf = torch.empty((N * F, pub.ct_words), dtype=torch.int32, device=dev)
        i = torch.arange(N, dtype=torch.int64, device=dev)
        idx = torch.cat([i * F + f for f in range(F)])
        offs = torch.arange(F + 1, dtype=torch.int64, device=dev) * N
        agg = torch.empty((F, pub.ct_words), dtype=torch.int32, device=dev)
        rep = torch.arange(N * F, dtype=torch.int64, device=dev) // F
        # feature-major entries for the multi-exponentiation: entry (f, i) -> ciphertext i, exponent x_if
        iF = torch.arange(N, dtype=torch.int64, device=dev).repeat(F)
        txf = torch.from_numpy(np.ascontiguousarray(x.T).reshape(N * F, 1).view(np.int32)).to(dev)

        def step(s):
            mark("t0")
            flb.pack(pub, cd, td, out=pt)
            mark("pack")
            if args.encrypt == "keyholder":
                flb.encrypt_crt(priv, pt, seed=s, out=ct)
            else:
                flb.encrypt(pub, pt, seed=s, out=ct)
            mark("encrypt")
            if os.environ.get("FLB_C3_NAIVE"):
                flb.scalar_mul(pub, ct.index_select(0, rep), tx, out=ctf)
                mark("scalar_mul")
                flb.reduce_segments(pub, ctf, offs, idx=idx, max_segment_len=N, out=agg)
            else:
                # per feature f: prod_i E(d_i)^(x_if) — segmented multi-exponentiation (Pippenger)
                flb.multiexp_segments(pub, ct, txf, offs, idx=iF, out=agg)
                mark("scalar_mul")
            mark("reduce")
            flb.decrypt(priv, agg)
            mark("decrypt")
        names = ["t0", "pack", "encrypt", "scalar_mul", "reduce", "decrypt"]
        ms, ph = run_steps(step, names)
        ops = N + N * F + N * F + F
        res.update(value=ops / (ms * 1e-3), ms_per_step=ms, breakdown_ms=ph,
                   ops_per_step={"encrypt": N, "scalar_mul": N * F, "add": N * F, "decrypt": F},
                   config={"workload": "C3 Hetero LR: 2048-bit key, 4,194,304 encrypted residuals (%s), "
                                       "x 8 u32 feature scalars each (scalar-mul), product per feature, "
                                       "decrypt 8" % args.encrypt, "key_bits": 2048,
                           "note": "scalar-mul + product per feature computed as one segmented "
                                   "multi-exponentiation (flb_multiexp_segments, Pippenger buckets; same result "
                                   "bits); ops_per_step counts the logical scalar-muls and adds. FLB_C3_NAIVE=1: "
                                   "explicit scalar_mul then reduce_segments"})
    elif wl == "c4":
        pub, priv = flb.keygen(2048, 0xF1B0 + 2048)
        nsamp, bins = 1 << 20, 256
        gh, bb, offsets, idx = synthetic.c4_histogram(n=nsamp, bins=bins)
        cd = flb.Codec(1.0, 44, 20, 2)
        tgh = torch.from_numpy(gh).to(dev)
        toff, tidx = torch.from_numpy(offsets).to(dev), torch.from_numpy(idx).to(dev)
        cnt = torch.from_numpy(np.diff(offsets).astype(np.int32)).to(dev)
        maxlen = int(np.diff(offsets).max())
        pt = torch.empty((nsamp, pub.pt_words), dtype=torch.int32, device=dev)
        ct = torch.empty((nsamp, pub.ct_words), dtype=torch.int32, device=dev)
        agg = torch.empty((bins, pub.ct_words), dtype=torch.int32, device=dev)

        def step(s):
            mark("t0")
            flb.pack(pub, cd, tgh, out=pt)
            mark("pack")
            if args.encrypt == "keyholder":
                flb.encrypt_crt(priv, pt, seed=s, out=ct)
            else:
                flb.encrypt(pub, pt, seed=s, out=ct)
            mark("encrypt")
            flb.reduce_segments(pub, ct, toff, idx=tidx, max_segment_len=maxlen, out=agg)
            mark("reduce")
            dd = flb.decrypt(priv, agg)
            mark("decrypt")
            flb.unpack(pub, cd, dd, 2 * bins, summands=cnt)
            mark("unpack")
        names = ["t0", "pack", "encrypt", "reduce", "decrypt", "unpack"]
        ms, ph = run_steps(step, names)
        ops = nsamp + (nsamp - bins) + bins
        res.update(value=ops / (ms * 1e-3), ms_per_step=ms, breakdown_ms=ph,
                   ops_per_step={"encrypt": nsamp, "add": nsamp - bins, "decrypt": bins},
                   config={"workload": "C4 Hetero SBT: 2048-bit key, 1,048,576 samples, (g, h) in two 64-bit "
                                       "slots (rho=44, b=20), encrypt (%s), segmented product into 256 "
                                       "quantile bins, decrypt 256, unpack with bin counts" % args.encrypt,
                           "key_bits": 2048})
    elif wl == "c5":
        per = {}
        for bits in (1024, 2048, 3072, 4096):
            M = args.c5_ops or ((1 << 20) if bits <= 2048 else (1 << 18))  # per rank (weak scaling)
            pub, priv = flb.keygen(bits, 0xF1B0 + bits)
            p, q, n = priv.export()
            base = synthetic.ints_to_limbs(synthetic.uniform_below(n, 256, 5 + bits), pub.pt_words).view(np.int32)
            m = torch.from_numpy(base).to(dev).repeat(M // 256, 1)
            c = torch.empty((M, pub.ct_words), dtype=torch.int32, device=dev)
            o = torch.empty_like(c)
            dm = torch.empty_like(m)
            ev.clear()

            def step(s):
                mark("t0")
                flb.encrypt(pub, m, seed=s, ctr0=rank * M, out=c)
                mark("enc")
                flb.encrypt_crt(priv, m, seed=s, ctr0=rank * M, out=o)
                mark("enc_crt")
                flb.decrypt(priv, c, out=dm)
                mark("dec")
                flb.add(pub, c, o, out=o)
                mark("add")
            names = ["t0", "enc", "enc_crt", "dec", "add"]
            ms, ph = run_steps(step, names)
            if world > 1:  # max over ranks of every phase (weak scaling: each rank its own batch)
                t = torch.tensor([ph[k] for k in names[1:]], dtype=torch.float64,
                                 device=dev if dist.get_backend() == "nccl" else "cpu")
                dist.all_reduce(t, op=dist.ReduceOp.MAX)
                ph = {k: float(t[i]) for i, k in enumerate(names[1:])}
            lp = {k: flb.op_cost(priv if k in ("decrypt", "encrypt_crt") else pub, k)[1]
                  for k in ("encrypt", "encrypt_crt", "decrypt", "add")}
            # tensor-core kernels: count the IMAD-pipe work they actually issue (op_cost 5/6/9)
            acct = {"encrypt": "cios", "encrypt_crt": "cios", "decrypt": "cios"}
            if os.environ.get("FLB_TC", "1") != "0":
                for k, tk, key in (("encrypt_crt", "encrypt_crt_tc", priv), ("decrypt", "decrypt_tc", priv),
                                   ("encrypt", "encrypt_tc", pub)):
                    try:
                        lp[k] = flb.op_cost(key, tk)[1]
                        acct[k] = "tensor-core (IMAD-pipe limb products of t = a b; reduction on tcgen05)"
                    except flb.FlbError:
                        pass
            peak = 148 * PEAK_LP_PER_CLK_SM * 1965e6
            W = world * M  # ops over all ranks
            per[str(bits)] = {
                "batch_per_rank": M,
                "encrypt_per_s": W / (ph["enc"] * 1e-3), "encrypt_keyholder_per_s": W / (ph["enc_crt"] * 1e-3),
                "decrypt_per_s": W / (ph["dec"] * 1e-3), "add_per_s": W / (ph["add"] * 1e-3),
                "frac_roofline": {"encrypt": lp["encrypt"] * W / (ph["enc"] * 1e-3) / peak / world,
                                  "encrypt_keyholder": lp["encrypt_crt"] * W / (ph["enc_crt"] * 1e-3) / peak / world,
                                  "decrypt": lp["decrypt"] * W / (ph["dec"] * 1e-3) / peak / world,
                                  "add": lp["add"] * W / (ph["add"] * 1e-3) / peak / world},
                "imad_accounting": acct}
            del c, o, dm, m
        v = per["2048"]
        res.update(value=3.0 / (1 / v["encrypt_per_s"] + 1 / v["decrypt_per_s"] + 1 / v["add_per_s"]),
                   ms_per_step=None, per_key=per,
                   n_gpus=world, scaling="weak",
                   config={"workload": "C5 key sweep 1024/2048/3072/4096: encrypt (public and key-holder), "
                                       "decrypt, add on uniform m < n; per rank batch 1,048,576 (1024/2048) and "
                                       "262,144 (3072/4096) per op instead of 16M (time budget; --c5-ops 16777216 "
                                       "runs the full batch), shard by ciphertext over %d rank(s)" % world,
                           "value_definition": "2048-bit enc/dec/add mix: 3 / sum of per-op seconds"})
    res["clocks"] = clk.stop()
    if rank == 0:
        print(json.dumps(res), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    if args.workload != "c2":
        return run_other(args)
    return run_flb(args)


if __name__ == "__main__":
    sys.exit(main())
