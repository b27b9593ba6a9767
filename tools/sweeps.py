"""SURVEY §8(d) diagnostics beside the headline (run on the GPU box; JSON lines to stdout):
  M2  sparsity sweep (Fig. 10 / line 252 analogue): the tile-sparse linear layer at M = 4096
      tokens for d x d (d = 768, 1024) and the BERT FFN shapes, tile ratio 0 ... 0.95;
  M3  sequence-length crossover (Fig. 8 / line 244 analogue): short vs long attention form vs the
      paper-literal partial OTF at fixed total tokens, BERT-base heads (H = 12, d_k = 64);
  M3b the same at batch 1 (Fig. 8's setting), BERT-base and Transformer heads;
  M4  pre-computed linear transformation vs the standard attention block (Fig. 9 / line 248-250).
Timing: CUDA events around 50 back-to-back launches after 5 warm-ups (operands L2-resident when they
fit: a kernel-level diagnostic, not the bench metric).  Dense torch.matmul at the same shape is
printed as context only (it is never a backend)."""
import json, math, os, sys
import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_chenhplg0d021_b200 as et  # noqa: E402
from et_synth import make_matrix  # noqa: E402

PEAK = {"hbm_gbs": 6547.5, "tc_tflops": 1642.5}
try:
    PEAK.update({k: v for k, v in json.load(open("MEASURED_PEAKS.json")).items() if k in ("hbm_gbs",)})
    PEAK["tc_tflops"] = json.load(open("MEASURED_PEAKS.json")).get("bf16_tflops", PEAK["tc_tflops"])
except Exception:
    pass


def timed(fn, reps=50, warm=5, graph=True):
    """Device time per call (us).  graph=True: `reps` calls captured in one CUDA graph and the graph
    replayed, so host launch overhead (ctypes + torch, several us per call) is not measured."""
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    if graph:
        g = torch.cuda.CUDAGraph()
        s = torch.cuda.Stream()
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s):
            with torch.cuda.graph(g, stream=s):
                for _ in range(reps):
                    fn()
        torch.cuda.current_stream().wait_stream(s)
        g.replay()
        torch.cuda.synchronize()
        run = g.replay
        n = reps
    else:
        run = lambda: [fn() for _ in range(reps)]
        n = reps
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record()
    run()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / n * 1e3   # us


def m2():
    M = 4096
    shapes = [("d768", 768, 768), ("d1024", 1024, 1024), ("ffn1", 3072, 768), ("ffn2", 768, 3072)]
    for name, N, K in shapes:
        W = torch.tensor(make_matrix(5, (N, K), 0.02, "fp16"), dtype=torch.float16, device="cuda")
        X = torch.tensor(make_matrix(6, (M, K), 1.0, "fp16"), dtype=torch.float16, device="cuda")
        dense_us = timed(lambda: torch.matmul(X, W.t()))
        for ratio in (0.0, 0.2, 0.4, 0.6, 0.8, 0.9, 0.95):
            pk = et.prune_pack(W, "tile", ratio)
            nnz = pk.c.ntiles
            epi = et.EPI_PART16 if K > 768 else et.EPI_BIAS
            out = et.linear_fwd(pk, X, None, epi)
            us = timed(lambda: et.linear_fwd(pk, X, None, epi, out=out))
            flops = 2.0 * M * 256 * nnz
            planes = (K + 767) // 768
            nbytes = M * K * 2 + nnz * 512 + M * N * 2 * planes
            print(json.dumps({"sweep": "M2", "shape": name, "M": M, "N": N, "K": K, "ratio": ratio, "kept_tiles": nnz,
                              "us": round(us, 2), "eff_tflops": round(flops / us / 1e6, 1),
                              "alg_gbs": round(nbytes / us / 1e3, 1),
                              "hbm_roofline_frac": round(nbytes / us / 1e3 / PEAK["hbm_gbs"], 3),
                              "dense_torch_matmul_us": round(dense_us, 2)}), flush=True)


def m2b():
    """Pruning-method comparison (Fig. 10 / line 252 analogue): tile vs row vs column
    pruned linear layer, d x d at M = 4096 tokens (S = 128, B = 32), ratio 0 ... 0.95.  Row: condensed
    output rows (padded to 16); column: X_adjusted gather + condensed-K tile GEMM (both launches
    timed)."""
    M = 4096
    for d in (768, 1024):
        W = torch.tensor(make_matrix(5, (d, d), 0.02, "fp16"), dtype=torch.float16, device="cuda")
        X = torch.tensor(make_matrix(6, (M, d), 1.0, "fp16"), dtype=torch.float16, device="cuda")
        dense_us = timed(lambda: torch.matmul(X, W.t()))
        for ratio in (0.0, 0.2, 0.4, 0.6, 0.8, 0.9, 0.95):
            row = {"sweep": "M2b", "d": d, "M": M, "ratio": ratio, "dense_torch_matmul_us": round(dense_us, 2)}
            epi = et.EPI_PART16 if d > 768 else et.EPI_BIAS
            pk = et.prune_pack(W, "tile", ratio)
            out = et.linear_fwd(pk, X, None, epi)
            row["tile_us"] = round(timed(lambda: et.linear_fwd(pk, X, None, epi, out=out)), 2)
            pr = et.prune_pack(W, "row", ratio)
            out_r = et.linear_fwd(pr, X, None, epi)
            row["row_us"] = round(timed(lambda: et.linear_fwd(pr, X, None, epi, out=out_r)), 2)
            cl = et.ColLinear(W, ratio)
            xa = torch.empty(M, cl.nk_pad, dtype=X.dtype, device="cuda")
            epi_c = et.EPI_PART16 if cl.nk_pad > 768 else et.EPI_BIAS
            out_c = et.linear_fwd(cl.dense, xa, None, epi_c)
            row["col_gather_us"] = round(timed(lambda: et.gather_cols(X, cl.keep, cl.nk_pad, out=xa)), 2)
            row["col_gemm_us"] = round(timed(lambda: et.linear_fwd(cl.dense, xa, None, epi_c, out=out_c)), 2)
            row["col_us"] = round(row["col_gather_us"] + row["col_gemm_us"], 2)
            row["col_kept"] = cl.nk
            print(json.dumps(row), flush=True)


def _m3_row(tag, S, B, H, dk):
    d = H * dk
    qkv = (torch.randn(B * S, 3 * d, device="cuda") * 0.5).half()
    Z = torch.empty(B * S, d, device="cuda").half()
    scores = torch.empty(et.attn_partial_scores_bytes(B, S, H, d, "fp16") // 2, dtype=torch.float16, device="cuda")
    flops = 4.0 * B * H * S * S * dk
    row = {"sweep": tag, "S": S, "B": B, "H": H, "d_k": dk}
    for mode in ("short", "long", "partial"):
        if mode == "short" and S > et.attn_short_max(dk):
            continue
        if mode == "partial":
            fn = lambda: et.attn_partial_fwd(qkv, B, S, H, d, 0, d, 2 * d, Z=Z, scores=scores)
        else:
            fn = lambda: et.attn_core_fwd(qkv, B, S, H, d, 0, d, 2 * d, mode=mode, scale=1.0, Z=Z)
        us = timed(fn)
        row[f"{mode}_us"] = round(us, 2)
        row[f"{mode}_eff_tflops"] = round(flops / us / 1e6, 1)
    fused = min(v for k, v in row.items() if k in ("short_us", "long_us"))
    row["partial_over_fused"] = round(row["partial_us"] / fused, 2)
    # the partial form's extra HBM traffic: the 16-bit score matrix written once, read twice
    row["partial_score_bytes"] = int(3 * B * H * S * S * 2)
    print(json.dumps(row), flush=True)


def m3():
    """Fixed total tokens (32768), BERT-base heads: the fused short / long forms vs the paper-literal
    partial OTF (et_attn_partial_fwd, NEXT-2)."""
    H, dk, total = 12, 64, 32768
    for S in (64, 128, 192, 224, 256, 320, 384, 512, 1024, 2048):
        _m3_row("M3", S, max(1, total // S), H, dk)


def m3b():
    """Fig. 8's own setting: one sequence, BERT-base (H = 12) and the
    Transformer (d_model 512, H = 8), S = 64 ... 2048 — latency-bound; where the paper's full OTF
    vs partial OTF crossover (224 on V100S) lands on B200."""
    for H in (12, 8):
        for S in (64, 128, 192, 224, 256, 320, 384, 512, 768, 1024, 2048):
            _m3_row("M3b", S, 1, H, 64)


def m4(batch=32):
    """Fig. 9 analogue (§5.2.3): the attention block (steps 1-8
    and the residual + LayerNorm) with vs without the pre-computed linear transformation, S = 128,
    d in {768, 1024, 2048}, heads with d_k in {64, 128}.  The paper prunes 50 % without and 80 % with
    the pre-computed operator (its accuracy budget); the 80 %-vs-80 % pair is printed too.  Without:
    W_Q/W_K/W_O tile, W_V row (attention-aware); with: W_Q/W_K tile, W_O row, W_V dense."""
    from et_synth import CONFIGS, make_layer, make_x
    S = 128
    for d in (768, 1024, 2048):
        for H in (d // 128, d // 64):
            cfg = CONFIGS["C2"].with_(d_model=d, heads=H, d_ff=4 * d, seq_len=S, batch=batch, layers=1)
            raw = make_layer(cfg, 0)
            X = torch.tensor(make_x(cfg).reshape(batch * S, d), dtype=torch.float16, device="cuda")
            row = {"sweep": "M4", "d": d, "H": H, "d_k": d // H, "S": S, "B": batch}
            for ratio in (0.5, 0.8):
                lay = et.pack_layer(raw, "attention-aware", ratio, H, "fp16")
                ws = torch.empty(et.attention_workspace_size(lay, batch, S, H, d, torch.float16), dtype=torch.uint8,
                                 device="cuda")
                out = torch.empty_like(X)
                row[f"std_{int(ratio * 100)}_us"] = round(timed(
                    lambda: et.attention_fwd(X, lay, batch, S, H, out=out, workspace=ws)), 2)
            pre = et.PreLayer(raw, 0.8, H, "fp16")
            wsp = torch.empty(pre.workspace_size(batch, S), dtype=torch.uint8, device="cuda")
            outp = torch.empty_like(X)
            row["pre_80_us"] = round(timed(lambda: pre(X, batch, S, out=outp, workspace=wsp)), 2)
            row["pre_Dv"] = pre.Dv
            row["speedup_pre80_vs_std50"] = round(row["std_50_us"] / row["pre_80_us"], 3)
            row["speedup_pre80_vs_std80"] = round(row["std_80_us"] / row["pre_80_us"], 3)
            print(json.dumps(row), flush=True)


if __name__ == "__main__":
    which = sys.argv[1:] or ["m2", "m2b", "m3", "m3b", "m4"]
    if "m2" in which:
        m2()
    if "m2b" in which:
        m2b()
    if "m3" in which:
        m3()
    if "m3b" in which:
        m3b()
    if "m4" in which:
        m4()
