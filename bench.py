#!/usr/bin/env python
"""bench.py — BERT-base encoder throughput of the B200-native E.T. hot path (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--config C3]

One step = one full forward of the workload's encoder stack over one batch of synthetic input
(SURVEY §8(a) rows a2-a7), through the library's public entry point et_encoder_fwd.

Workload (N=1): configs[2] = C3, BERT-base (12 layers, 12 heads, d_model 768, d_ff 3072), seq_len 128,
batch 32, 80 % tensor-tile pruning (16x16), FP16 — the configuration the metric is quoted on.
Multi-GPU (torchrun, one rank per GPU): the batch is sharded, every rank runs its own 32 sequences
(weak scaling, no collective on the data path; sequences are independent).

Timing: W untimed warm-up steps; then K steps, each bracketed by CUDA events on the launching stream,
L2 flushed (256 MiB write) before every step outside the events; barrier + synchronize around the
whole region; value = sequences of all ranks / max over ranks of the summed step time.  Per-kernel
times come from the library's trace events recorded live in the same timed steps (roofline).
`e2e` repeats the measurement through the same call with pinned-host input / output copies inside
the timed region, as a pipelined serving loop (H2D of step s+1 and D2H of step s-1 on two copy
streams overlap step s; flush and copies inside one event pair over all K steps); `serial_value` is
the same with copy -> forward -> copy in series per step.  `cpu_baseline`: the float64 CPU oracle (tests' reference; never the product path)
on a bounded sample, rank 0 at N=1 only.  `--impl reference`: that oracle as the reference arm.
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

import numpy as np  # noqa: E402

METRIC = "BERT-base encoder seqs/sec @seq128, 80% tile-pruned; % tensor-pipe/HBM roofline"
KIND_NAMES = ["qkv_gemm", "attention", "oproj_gemm", "ln1", "ffn1_gemm", "ffn2_gemm", "ln2", "aux"]
SPEC_TC_TFLOPS = 2250.0


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", default="C3")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-parity", action="store_true", help="skip the sampled oracle comparison in the line")
    ap.add_argument("--cpu-seconds", type=float, default=12.0, help="budget of the cpu_baseline sample")
    ap.add_argument("--scaling", choices=["weak", "strong"], default=None,
                    help="weak: every rank runs the config's batch (default; C3 metric); strong: the config's "
                         "batch is the global batch, split over the ranks (default for C5: B = 256 / N)")
    ap.add_argument("--parallel", choices=["batch", "head"], default="batch",
                    help="batch: batch sharding (default, weak scaling); head: head-parallel latency mode "
                         "(Eq. 4 partials + NCCL all-reduce per layer, strong scaling)")
    return ap.parse_args()


def peaks():
    p = {"hbm_gbs": 6482.1, "bf16_tflops": 1637.3, "bf16_tflops_sustained": 1384.3, "src": "MEASURED_PEAKS.json"}
    f = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(f):
        with open(f) as fh:
            m = json.load(fh)
        for k in ("hbm_gbs", "bf16_tflops", "bf16_tflops_sustained"):
            if k in m:
                p[k] = float(m[k])
    else:
        p.update({"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0,
                  "src": "fallback (B200_PROFILING.md)"})
    return p


# ------------------------------------------------------------------------------------------ clocks
class ClockSampler:
    """SM clock / power / clock-event-reason sampling DURING the timed region (B200_PROFILING.md
    clocks line).  NVML polled every 2 ms from a thread (the timed region is ~0.1-0.2 s, shorter
    than nvidia-smi's sampling period); nvidia-smi -lms 100 as the fallback."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
    BITS = {"sw_power_cap": 0x4, "hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20,
            "hw_thermal_slowdown": 0x40, "hw_power_brake_slowdown": 0x80}

    def __init__(self, gpu_index: int):
        self.idx = gpu_index
        self.proc = None
        self.lines = []
        self.samples = []
        self.stop_ev = threading.Event()
        self.nvml = None
        try:
            import pynvml
            pynvml.nvmlInit()
            h = None
            try:
                import torch
                # torch's pci_* properties are integers: match them against every NVML device
                pr = torch.cuda.get_device_properties(gpu_index)
                for i in range(pynvml.nvmlDeviceGetCount()):
                    hi = pynvml.nvmlDeviceGetHandleByIndex(i)
                    pci = pynvml.nvmlDeviceGetPciInfo(hi)
                    if (pci.bus, pci.device, pci.domain) == (pr.pci_bus_id, pr.pci_device_id, pr.pci_domain_id):
                        h = hi
                        break
                if h is None:
                    raise RuntimeError("no NVML device matches the CUDA device")
            except Exception:
                h = pynvml.nvmlDeviceGetHandleByIndex(gpu_index)
            self.nvml, self.h = pynvml, h
            self.max_mhz = float(pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM))
        except Exception:
            self.nvml = None

    def _poll(self):
        nv, h = self.nvml, self.h
        while not self.stop_ev.is_set():
            try:
                self.samples.append((float(nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)),
                                     int(nv.nvmlDeviceGetCurrentClocksEventReasons(h)),
                                     nv.nvmlDeviceGetPowerUsage(h) / 1000.0))
            except Exception:
                pass
            time.sleep(0.002)

    def start(self, wait_first: float = 3.0):
        if self.nvml is not None:
            self.t = threading.Thread(target=self._poll, daemon=True)
            self.t.start()
            return
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.idx}", f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
            t0 = time.time()
            while not self.lines and time.time() - t0 < wait_first:   # sampler live before timing
                time.sleep(0.02)
            self.lines.clear()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.nvml is not None:
            self.stop_ev.set()
            self.t.join(timeout=1)
            sm = [s[0] for s in self.samples]
            reasons = {n for n, bit in self.BITS.items() for s in self.samples if s[1] & bit}
            load = [x for x in sm if x > 300] or sm
            return {"sm_mhz": statistics.median(load) if load else None, "sm_max_mhz": self.max_mhz,
                    "reasons": sorted(reasons), "samples": len(sm),
                    "power_w_max": max(s[2] for s in self.samples) if self.samples else None, "source": "nvml"}
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, mx, reasons, pw = [], [], set(), []
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx.append(float(f[2]))
                pw.append(float(f[3]))
            except ValueError:
                continue
            for n, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(n)
        load = [s for s in sm if s > 300] or sm
        return {"sm_mhz": statistics.median(load) if load else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm), "power_w_max": max(pw) if pw else None,
                "source": "nvidia-smi"}


# ------------------------------------------------------------------------------------------ roofline model
STEP_OF_KERNEL = {"qkv_gemm": "qkv", "attention": "attention", "oproj_gemm": "oproj_ln", "ln1": "oproj_ln",
                  "ffn1_gemm": "ffn1", "ffn2_gemm": "ffn2_ln", "ln2": "ffn2_ln"}


def step_model(cfg, nnz: dict, v_kept: int | None, es: int):
    """algorithmic bytes and effective FLOPs of one layer's five steps
    (whole batch).  Bytes = read the step's inputs + its kept weights + write its outputs once, in the
    storage dtype (es bytes; the residual stream counted like the activations, as in Appendix B);
    FLOPs = 2 M x kept weights (16x16 tiles, or kept W_V rows) + attention on unmasked (q, k) pairs,
    P.V over the kept V features.  nnz: kept tiles per tile-pruned matrix; v_kept: kept W_V rows when
    W_V is row-pruned (else None)."""
    M, d, f, H, S, B = cfg.tokens, cfg.d_model, cfg.d_ff, cfg.heads, cfg.seq_len, cfg.batch
    dk = d // H
    t = 256 * es                                      # bytes of one kept 16x16 tile
    mm = lambda n: 2.0 * M * 256 * n                 # noqa: E731  one tile against M tokens
    pairs = B * (S * (S + 1) / 2 if cfg.causal else S * S)   # unmasked (q, k) pairs per head (lengths = S)
    vw = v_kept if v_kept is not None else d          # V width the attention moves / multiplies
    wv_b = v_kept * d * es if v_kept is not None else nnz["wv"] * t
    wv_f = 2.0 * M * v_kept * d if v_kept is not None else mm(nnz["wv"])
    return {
        "qkv": (M * d * es + (nnz["wq"] + nnz["wk"]) * t + wv_b + M * (2 * d + vw) * es,
                mm(nnz["wq"] + nnz["wk"]) + wv_f),
        "attention": (M * (2 * d + vw) * es + M * d * es, 2.0 * pairs * H * dk + 2.0 * pairs * vw),
        "oproj_ln": (M * d * es + nnz["wo"] * t + M * d * es + M * d * es, mm(nnz["wo"])),
        "ffn1": (M * d * es + nnz["w1"] * t + M * f * es, mm(nnz["w1"])),
        "ffn2_ln": (M * f * es + nnz["w2"] * t + M * d * es + M * d * es, mm(nnz["w2"])),
    }


# ------------------------------------------------------------------------------------------ CPU oracle
def oracle_seqs_per_s(cfg, raws, X, lens, budget_s: float, chunk: int):
    """Time the float64 CPU oracle (as it stands) on chunks of `chunk` sequences until the budget."""
    from oracle import encoder as oe
    layers = [oe.prune_layer(r, cfg.scheme, cfg.ratio)[0] for r in raws]
    done, t0 = 0, time.perf_counter()
    while True:
        i0 = done % cfg.batch
        idx = np.arange(i0, i0 + chunk) % cfg.batch
        oe.encoder(X[idx].astype(np.float64), layers, cfg.heads, lens[idx], cfg.causal, cfg.act, cfg.ln_eps)
        done += chunk
        el = time.perf_counter() - t0
        if el >= budget_s:
            return done / el, done, el


def parity_sample(cfg, raws, X, lens, Y, layers_packed, nseq: int = 2):
    """SURVEY §8(d) line fields: the GPU output of the first `nseq` sequences of the timed batch
    against the float64 oracle (max-abs, relative Frobenius), and layer 0's six packed masks against
    the oracle's selection (bit-exact).  Test infrastructure only: it runs after the timed regions."""
    from oracle import encoder as oe
    nseq = min(nseq, cfg.batch)
    pruned = [oe.prune_layer(r, cfg.scheme, cfg.ratio) for r in raws]
    ref = oe.encoder(X[:nseq].astype(np.float64), [p[0] for p in pruned], cfg.heads, lens[:nseq], cfg.causal,
                     cfg.act, cfg.ln_eps).reshape(nseq * cfg.seq_len, cfg.d_model)
    got = Y[: nseq * cfg.seq_len].float().cpu().numpy().astype(np.float64)
    d = got - ref
    masks_ok = True
    for n in ("wq", "wk", "wv", "wo", "w1", "w2"):
        want = pruned[0][1][n]["mask"]
        have = layers_packed[0].packed[n].mask().cpu().numpy().view(np.uint32)[: want.size]
        masks_ok = masks_ok and bool(np.array_equal(have, want))
    return {"sequences": nseq, "max_abs": float(np.abs(d).max()),
            "rel_fro": float(np.linalg.norm(d) / np.linalg.norm(ref)), "tol_max_abs": 2e-2, "tol_rel_fro": 5e-3,
            "masks_bit_exact_layer0": masks_ok}


def git_sha():
    """The revision libet.so was built from (build/BUILD_SHA, written by build.py), else git."""
    try:
        with open(os.path.join(ROOT, "build", "BUILD_SHA")) as fh:
            return fh.read().strip() or None
    except OSError:
        pass
    try:
        return subprocess.run(["git", "rev-parse", "--short", "HEAD"], cwd=ROOT, capture_output=True, text=True,
                              timeout=5).stdout.strip() or None
    except Exception:
        return None


def cpu_threads():
    try:
        from threadpoolctl import threadpool_info
        n = [i.get("num_threads") for i in threadpool_info() if i.get("user_api") == "blas"]
        if n:
            return int(max(n))
    except Exception:
        pass
    return os.cpu_count()


def reference_arm(args):
    """--impl reference: the CPU oracle on the same config/metric (bounded sample per step)."""
    from et_synth import CONFIGS, make_layer, make_lengths, make_x
    cfg = CONFIGS[args.config]
    raws = [make_layer(cfg, l) for l in range(cfg.layers)]
    X = make_x(cfg)
    lens = make_lengths(cfg, ragged=False)
    from oracle import encoder as oe
    layers = [oe.prune_layer(r, cfg.scheme, cfg.ratio)[0] for r in raws]
    per_step = 1 if cfg.seq_len > 512 else 2
    for w in range(args.warmup):
        idx = np.arange(w * per_step, (w + 1) * per_step) % cfg.batch
        oe.encoder(X[idx].astype(np.float64), layers, cfg.heads, lens[idx], cfg.causal, cfg.act, cfg.ln_eps)
    t0 = time.perf_counter()
    for s in range(args.steps):
        idx = np.arange(s * per_step, (s + 1) * per_step) % cfg.batch
        oe.encoder(X[idx].astype(np.float64), layers, cfg.heads, lens[idx], cfg.causal, cfg.act, cfg.ln_eps)
    el = time.perf_counter() - t0
    v = per_step * args.steps / el
    sample = f"{per_step} sequences of {args.config} per step (float64 numpy, all {cfg.layers} layers)"
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "seqs/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * el / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": workload_name(cfg), "global_batch": cfg.batch, "seq_len": cfg.seq_len},
            "cpu_baseline": {"value": v, "unit": "seqs/s", "cores": cpu_threads(), "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": v, "unit": "seqs/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def workload_name(cfg):
    return (f"{cfg.name}: {cfg.layers}-layer encoder, {cfg.heads} heads, d_model {cfg.d_model}, d_ff {cfg.d_ff}, "
            f"seq_len {cfg.seq_len}, {cfg.ratio:.0%} {cfg.scheme} pruning (16x16 tiles), {cfg.dtype}, "
            f"{'causal' if cfg.causal else 'padding'} mask")


# ------------------------------------------------------------------------------------------ our arm
def our_arm(args):
    import torch
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if not torch.cuda.is_available():
        raise SystemExit("bench.py: no CUDA device (this benchmark has no CPU fallback)")
    torch.cuda.set_device(local)
    dist = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    import paper_conf_sc_chenhplg0d021_b200 as et
    from et_synth import CONFIGS, make_layer, make_lengths, make_x

    from paper_conf_sc_chenhplg0d021_b200.dist import shard_range
    base = CONFIGS[args.config]
    strong = (args.scaling == "strong") if args.scaling else base.name == "C5"
    if strong:   # the config's batch is the global batch (C5: 256 sequences over N GPUs)
        if base.batch % world:
            raise SystemExit(f"bench.py: global batch {base.batch} does not split over {world} ranks")
        cfg, gcfg = base.with_(batch=base.batch // world), base
    else:        # every rank runs the config's batch
        cfg, gcfg = base, base.with_(batch=base.batch * world)
    dtype = cfg.dtype                            # C1: fp32 (the validation build, its BASELINE precision)
    rdt = dtype if cfg.resid == "same" else cfg.resid   # residual-stream dtype (reading C-22)
    raws = [make_layer(cfg, l) for l in range(cfg.layers)]
    Xg = make_x(gcfg)
    b0, b1 = shard_range(gcfg.batch, world, rank)
    X = Xg[b0:b1]
    lens = make_lengths(cfg, ragged=False)

    layers = [et.pack_layer(r, cfg.scheme, cfg.ratio, cfg.heads, dtype) for r in raws]
    if world > 1:   # every rank packed the same masks (deterministic pack): checked, not assumed
        from paper_conf_sc_chenhplg0d021_b200.dist import all_equal_across_ranks, layers_digest
        if not all_equal_across_ranks(layers_digest(layers)):
            raise SystemExit("bench.py: ranks packed different masks")
    # kept 16x16 tiles per tile-pruned matrix; kept W_V rows (not padded tiles) when row-pruned
    nnz_layers = [{n: l.packed[n].c.nnz for n in ("wq", "wk", "wv", "wo", "w1", "w2")} for l in layers]
    vkept_layers = [l.packed["wv"].c.nnz if cfg.scheme == "attention-aware" else None for l in layers]
    L = torch.from_numpy(lens).cuda()
    enc = et.Encoder(layers, cfg.batch, cfg.seq_len, cfg.heads, cfg.d_ff, act=cfg.act, ln_eps=cfg.ln_eps,
                     dtype=dtype, resid_dtype=rdt, causal=cfg.causal, mode=cfg.attn_mode, lengths=L)
    tdt = et.torch_dtype(rdt)
    Xd = torch.from_numpy(np.ascontiguousarray(X.reshape(cfg.tokens, cfg.d_model))).cuda().to(tdt)
    out = torch.empty_like(Xd)
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    stream = torch.cuda.current_stream()

    def barrier():
        if dist is not None:
            dist.barrier()

    for _ in range(3):   # eager calls: first-use kernel attributes, tensor-map encoder
        enc(Xd, out)
    torch.cuda.synchronize()
    # the forward as one CUDA graph (et_encoder_graph_create): the timed unit is one replay
    graph = enc.capture(Xd, out)
    K = args.steps
    cap = len(layers) * 8 + 4
    slots = torch.empty(2 * cap, dtype=torch.int64, device="cuda")   # device-side kernel spans (et.h tracing)
    et._check(et._lib.et_trace_begin(cap, slots.data_ptr()))
    graph_tr = enc.capture(Xd, out)       # same kernels, each stamping its device span into `slots`
    n_int = __import__("ctypes").c_int32()
    et._check(et._lib.et_trace_end(__import__("ctypes").byref(n_int)))
    for _ in range(max(args.warmup, 3)):
        graph.launch()
    torch.cuda.synchronize()

    # ---------------- timed region: K steps (graph replays), per-step events, L2 flushed between steps
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    clk = ClockSampler(local)
    barrier()
    torch.cuda.synchronize()
    clk.start()
    launches0 = et._lib.et_launch_count()
    for s in range(K):
        flush.fill_(float(s))
        ev[s][0].record(stream)
        graph.launch()
        ev[s][1].record(stream)
    launches = et._lib.et_launch_count() - launches0
    torch.cuda.synchronize()
    barrier()
    clocks = clk.stop()
    step_ms = [a.elapsed_time(b) for a, b in ev]
    t_local = sum(step_ms) / 1e3

    # ---------------- per-kernel device time: K replays of the traced graph, same flush discipline
    # (every kernel's span = first CTA start to last CTA end, from %globaltimer inside the kernels)
    import ctypes
    kind = ctypes.c_int32()
    ms = ctypes.c_float()
    per_kind = {}
    tr_ms = []
    for s in range(K):
        flush.fill_(float(s))
        slots.fill_(-1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        graph_tr.launch()
        e1.record(stream)
        torch.cuda.synchronize()
        tr_ms.append(e0.elapsed_time(e1))
        for i in range(n_int.value):
            et._check(et._lib.et_trace_get(i, ctypes.byref(kind), ctypes.byref(ms)))
            if kind.value < len(KIND_NAMES):
                per_kind.setdefault(KIND_NAMES[kind.value], []).append(ms.value)

    # ---------------- end to end: pinned host input -> device, graph replay, device -> pinned host output
    e2e = None
    if not args.no_e2e:
        Xh = torch.from_numpy(np.ascontiguousarray(X.reshape(cfg.tokens, cfg.d_model))).to(tdt).pin_memory()
        Oh = torch.empty_like(Xh).pin_memory()
        eev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
        for _ in range(2):
            Xd.copy_(Xh, non_blocking=True)
            graph.launch()
            Oh.copy_(out, non_blocking=True)
        torch.cuda.synchronize()
        barrier()
        for s in range(K):
            flush.fill_(float(s))
            eev[s][0].record(stream)
            Xd.copy_(Xh, non_blocking=True)
            graph.launch()
            Oh.copy_(out, non_blocking=True)
            eev[s][1].record(stream)
        torch.cuda.synchronize()
        barrier()
        e2e_serial = sum(a.elapsed_time(b) for a, b in eev) / 1e3
        # pipelined serving loop (the same calls): two input / output buffer pairs, each with its own
        # captured graph; the H2D copy of step s+1 and the D2H copy of step s-1 run on two copy streams
        # while step s computes.  Every step's copies and the L2 flush are inside the timed region
        # (one event pair around all K steps, the copy streams joined before the end event).
        Xd_b, out_b = torch.empty_like(Xd), torch.empty_like(out)
        graphs = [graph, enc.capture(Xd_b, out_b)]
        xin, xout = [Xd, Xd_b], [out, out_b]
        Oh2 = [Oh, torch.empty_like(Oh).pin_memory()]
        s_in, s_out = torch.cuda.Stream(), torch.cuda.Stream()
        comp_done = [torch.cuda.Event() for _ in range(2)]
        in_ready = [torch.cuda.Event() for _ in range(2)]
        out_free = [torch.cuda.Event() for _ in range(2)]
        for e in comp_done + out_free:
            e.record(stream)
        torch.cuda.synchronize()
        barrier()
        p0, p1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        p0.record(stream)
        s_in.wait_stream(stream)
        s_out.wait_stream(stream)
        for st in range(K):
            i = st % 2
            with torch.cuda.stream(s_in):
                s_in.wait_event(comp_done[i])          # step st-2 has finished reading xin[i]
                xin[i].copy_(Xh, non_blocking=True)
                in_ready[i].record(s_in)
            stream.wait_event(in_ready[i])
            stream.wait_event(out_free[i])             # the D2H of step st-2 has read xout[i]
            flush.fill_(float(st))
            graphs[i].launch()
            comp_done[i].record(stream)
            with torch.cuda.stream(s_out):
                s_out.wait_event(comp_done[i])
                Oh2[i].copy_(xout[i], non_blocking=True)
                out_free[i].record(s_out)
        stream.wait_stream(s_in)
        stream.wait_stream(s_out)
        p1.record(stream)
        torch.cuda.synchronize()
        barrier()
        e2e_local = p0.elapsed_time(p1) / 1e3
        e2e = {"t": e2e_local, "h2d": Xh.numel() * Xh.element_size(), "d2h": Oh.numel() * Oh.element_size(),
               "serial_t": e2e_serial}

    # ---------------- max over ranks
    t_max = t_local
    e2e_max = e2e["t"] if e2e else None
    if dist is not None:
        tt = torch.tensor([t_local, e2e_max or 0.0], dtype=torch.float64, device="cuda")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        t_max, e2e_max = float(tt[0]), (float(tt[1]) if e2e else None)

    if rank == 0:
        pk = peaks()
        total_seqs = cfg.batch * world * K
        value = total_seqs / t_max
        es = 4 if dtype == "fp32" else 2
        models = [step_model(cfg, nz, vk, es) for nz, vk in zip(nnz_layers, vkept_layers)]
        # dominant kernel: largest share of the traced step time; its SURVEY §8(d) step's algorithmic
        # bytes / FLOPs over the step's kernels' average device spans (the O-projection and FFN2 steps
        # include their LayerNorm kernel: "O proj + res + LN", "FFN2 + res + LN")
        tot = {k: sum(v) for k, v in per_kind.items()}
        dom = max(tot, key=tot.get) if tot else None
        roof = None
        if dom and dom in STEP_OF_KERNEL:
            step = STEP_OF_KERNEL[dom]
            kerns = [k for k, st in STEP_OF_KERNEL.items() if st == step and k in per_kind]
            avg_s = sum(statistics.mean(per_kind[k]) for k in kerns) / 1e3
            nbytes, nflops = models[0][step]
            t_hbm = nbytes / (pk["hbm_gbs"] * 1e9)
            t_tc = nflops / (pk["bf16_tflops"] * 1e12)
            traffic = None
            tf = os.path.join(ROOT, "profiles", "ncu_traffic.json")
            if os.path.exists(tf):
                with open(tf) as fh:
                    tj = json.load(fh)
                if all(k in tj for k in kerns):
                    traffic = sum(tj[k] for k in kerns)
            name = "+".join(kerns)
            if dtype == "fp32":   # the validation build runs on the CUDA cores: report the HBM line
                t_tc = 0.0
            if t_tc > t_hbm:
                ach = nflops / avg_s / 1e12
                roof = {"bound": "tensor", "achieved": ach, "peak": pk["bf16_tflops"], "unit": "TFLOP/s",
                        "frac": ach / pk["bf16_tflops"], "traffic": traffic, "kernel": name, "step": step,
                        "algorithmic_flops_per_launch": nflops, "avg_launch_ms": avg_s * 1e3,
                        "peak_src": pk["src"] + " bf16_tflops (burst; fp16 dense = bf16 dense)"}
            else:
                ach = nbytes / avg_s / 1e9
                roof = {"bound": "hbm", "achieved": ach, "peak": pk["hbm_gbs"], "unit": "GB/s",
                        "frac": ach / pk["hbm_gbs"], "traffic": traffic, "kernel": name, "step": step,
                        "algorithmic_bytes_per_launch": nbytes, "avg_launch_ms": avg_s * 1e3,
                        "peak_src": pk["src"] + " hbm_gbs"}
        share = {k: round(v / sum(tot.values()), 4) for k, v in tot.items()} if tot else {}
        kern_ms = {k: round(statistics.mean(v), 5) for k, v in per_kind.items()}
        # stepwise roofline: sum over layers and steps of max(F / P_tc, B / P_hbm),
        # on the algorithmic bytes of Appendix B, divided by the measured step time
        t_roof = sum(max(f / (pk["bf16_tflops"] * 1e12), b / (pk["hbm_gbs"] * 1e9))
                     for m in models for b, f in m.values())
        eflops = sum(f for m in models for _, f in m.values()) * world
        ns = {"eff_gflop_per_step": eflops / 1e9, "eff_tflops": eflops * K / t_max / 1e12}
        ns["frac_of_measured_tc_burst"] = ns["eff_tflops"] / pk["bf16_tflops"]
        ns["frac_of_measured_tc_sustained"] = ns["eff_tflops"] / pk["bf16_tflops_sustained"]
        ns["frac_of_spec_tc"] = ns["eff_tflops"] / SPEC_TC_TFLOPS
        ns["target_frac"] = 0.60
        line = {
            "metric": METRIC, "value": value, "unit": "seqs/s", "n_gpus": world, "steps": K,
            "warmup": max(args.warmup, 3), "ms_per_step": 1e3 * t_max / K, "higher_is_better": True,
            "scaling": "strong" if strong else "weak", "vs_baseline": None, "dtype": dtype, "data": "synthetic",
            "config": {"workload": workload_name(gcfg if strong else cfg), "global_batch": cfg.batch * world,
                       "seq_len": cfg.seq_len, "per_gpu_batch": cfg.batch,
                       "parallelism": f"dp{world} (batch sharded, no data-path collective)",
                       "l2": "flushed before every timed step (256 MiB write, outside the events)",
                       "residual_stream": rdt, "attention_form": "short" if cfg.seq_len <= 256 else "long"},
            "roofline": roof,
            "kernel_ms": kern_ms, "kernel_share": share,
            "north_star": ns,
            "gpu_launches": int(launches),
            "clocks": clocks,
            "step_ms_p50": statistics.median(step_ms),
            "step_ms_p10": float(np.percentile(step_ms, 10)), "step_ms_p90": float(np.percentile(step_ms, 90)),
            "stepwise_roofline_frac": t_roof / (t_max / K),
            "stepwise_roofline_ms": t_roof * 1e3,
            "stepwise_bytes_per_layer": sum(b for b, _ in models[0].values()),
            "git": git_sha(),
            "traced_step_ms_p50": statistics.median(tr_ms),
            "launch": "one CUDA graph replay per step (et_encoder_graph_create / et_graph_launch)",
        }
        if e2e:
            line["e2e"] = {"value": total_seqs / e2e_max, "unit": "seqs/s", "h2d_bytes_per_step": e2e["h2d"],
                           "d2h_bytes_per_step": e2e["d2h"],
                           "mode": "pipelined: H2D of step s+1 / D2H of step s-1 on copy streams overlap step s; "
                                   "L2 flush and all copies inside one timed region over K steps",
                           "serial_value": total_seqs / e2e["serial_t"]}
        if not args.no_parity:
            line["parity"] = parity_sample(cfg, raws, X, lens, out, layers)
        if world == 1 and not args.no_cpu_baseline:
            v, n, el = oracle_seqs_per_s(cfg, raws, X, lens, args.cpu_seconds, chunk=1 if cfg.seq_len > 512 else 2)
            line["cpu_baseline"] = {"value": v, "unit": "seqs/s", "cores": cpu_threads(), "kind": "oracle",
                                    "sample": f"{n} sequences of {args.config} (all {cfg.layers} layers, float64 "
                                              f"numpy oracle, {el:.1f} s)"}
        print(json.dumps(line), flush=True)
    if dist is not None:
        dist.barrier()
        dist.destroy_process_group()


# ------------------------------------------------------------------------------------------ head-parallel arm
def head_parallel_arm(args):
    """Head-parallel latency mode: every rank runs the whole batch on its heads
    (dist.HeadParallelEncoder), an NCCL all-reduce of the FP32 O-projection partials per layer, the
    FFN replicated.  Total work fixed as N grows ("strong").  Eager launches (the all-reduce sits
    between library calls), so this mode is host-launch bound at small batches."""
    import torch
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if not torch.cuda.is_available():
        raise SystemExit("bench.py: no CUDA device (this benchmark has no CPU fallback)")
    torch.cuda.set_device(local)
    import torch.distributed as dist
    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    os.environ.setdefault("MASTER_PORT", "29518")
    if not dist.is_initialized():
        dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda", local))
    import paper_conf_sc_chenhplg0d021_b200 as et
    from et_synth import CONFIGS, make_layer, make_lengths, make_x
    from paper_conf_sc_chenhplg0d021_b200.dist import HeadParallelEncoder
    cfg = CONFIGS[args.config]
    dtype = cfg.dtype if cfg.dtype != "fp32" else "fp16"
    raws = [make_layer(cfg, l) for l in range(cfg.layers)]
    layers = [et.pack_layer(r, cfg.scheme, cfg.ratio, cfg.heads, dtype) for r in raws]
    L = torch.from_numpy(make_lengths(cfg, ragged=False)).cuda()
    enc = HeadParallelEncoder(raws, layers, cfg.heads, cfg.batch, cfg.seq_len, cfg.d_ff, act=cfg.act,
                              ln_eps=cfg.ln_eps, dtype=dtype, causal=cfg.causal, mode=cfg.attn_mode, lengths=L,
                              rank=rank, world=world, group=dist.group.WORLD)
    X = make_x(cfg)
    Xd = torch.from_numpy(np.ascontiguousarray(X.reshape(cfg.tokens, cfg.d_model))).cuda().to(et.torch_dtype(dtype))
    out = torch.empty_like(Xd)
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    stream = torch.cuda.current_stream()
    for _ in range(max(args.warmup, 3)):
        enc(Xd, out)
    torch.cuda.synchronize()
    K = args.steps

    def timed(step):
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
        dist.barrier()
        torch.cuda.synchronize()
        for s in range(K):
            flush.fill_(float(s))
            ev[s][0].record(stream)
            step()
            ev[s][1].record(stream)
        torch.cuda.synchronize()
        dist.barrier()
        t = torch.tensor([sum(a.elapsed_time(b) for a, b in ev) / 1e3], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t[0])

    l0 = et._lib.et_launch_count()
    enc(Xd, out)
    per_fwd = et._lib.et_launch_count() - l0
    t_eager = timed(lambda: enc(Xd, out))
    # the whole forward (12 layers x library kernels + 12 NCCL all-reduces) as one CUDA graph
    graph = enc.capture(Xd, out)
    for _ in range(3):
        graph.replay()
    clk = ClockSampler(local)
    clk.start()
    t_max = timed(graph.replay)
    clocks = clk.stop()
    launches = per_fwd * K
    if rank == 0:
        line = {
            "metric": METRIC, "value": cfg.batch * K / t_max, "unit": "seqs/s", "n_gpus": world, "steps": K,
            "warmup": max(args.warmup, 3), "ms_per_step": 1e3 * t_max / K, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": dtype, "data": "synthetic",
            "config": {"workload": workload_name(cfg), "global_batch": cfg.batch, "seq_len": cfg.seq_len,
                       "parallelism": f"hp{world} (head-parallel: W_O partials + NCCL all-reduce per layer, "
                                      f"FFN replicated)",
                       "heads_rank0": [enc.h0, enc.h1],
                       "l2": "flushed before every timed step (256 MiB write, outside the events)",
                       "launch": "one CUDA graph per forward (library kernels + NCCL all-reduces captured)"},
            "gpu_launches": int(launches), "clocks": clocks, "mode": "head-parallel (latency mode, optional)",
            "eager_value": cfg.batch * K / t_eager,
        }
        print(json.dumps(line), flush=True)
    dist.barrier()
    dist.destroy_process_group()


def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if args.impl == "reference":
        if int(os.environ.get("RANK", "0")) == 0:
            reference_arm(args)
        return
    if args.gpus > 1 and world == 1 and "RANK" not in os.environ:
        # launched directly with --gpus N: re-launch one process per GPU through torchrun
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr", "127.0.0.1", "--master-port", "29517", __file__] + sys.argv[1:]
        raise SystemExit(subprocess.call(cmd))
    if args.parallel == "head":
        head_parallel_arm(args)
        return
    our_arm(args)


if __name__ == "__main__":
    main()
