"""Head-parallel mode (Eq. 4: Output = sum_h Z_h W_O,h^T) on one
GPU: the ranks' partials are computed one after another on cuda:0 and summed (the all-reduce's
arithmetic), then compared with the float64 oracle and with the single-call full-range block.
The NCCL exchange itself runs in test_head_parallel_encoder_nccl (world size 1 on one GPU; the
multi-rank exchange is covered on CPU by tests/test_dist_cpu.py over gloo)."""
import os
import socket

import numpy as np
import pytest
import torch

from et_synth import CONFIGS, make_layer, make_lengths, make_x
from oracle import encoder as oe
from tests.gpu_util import assert_close, dev_tensor, to64

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def etm():
    import paper_conf_sc_chenhplg0d021_b200 as m
    assert torch.cuda.is_available()
    return m


def _case(key, **kw):
    cfg = CONFIGS[key].with_(**kw)
    raws = [make_layer(cfg, l) for l in range(cfg.layers)]
    return cfg, raws, make_x(cfg), make_lengths(cfg)


@pytest.mark.parametrize("key,kw,worlds", [
    ("C3", {"layers": 1, "batch": 2}, (2, 3, 8)),          # tile, d_k 64, 12 heads (8 ranks: 2/1 imbalance)
    ("C2", {}, (2, 4)),                                    # attention-aware (W_V row), d_k 128, causal
    ("C3", {"layers": 1, "batch": 2, "dtype": "bf16"}, (2,)),
    ("C4", {"layers": 1, "batch": 1, "seq_len": 384}, (3,)),   # attention-aware, long form
])
def test_head_parallel_partials_sum_to_full_block(etm, key, kw, worlds):
    from paper_conf_sc_chenhplg0d021_b200.dist import head_range, pack_head_slice
    cfg, raws, X, lens = _case(key, **kw)
    raw = raws[0]
    full = etm.pack_layer(raw, cfg.scheme, cfg.ratio, cfg.heads, cfg.dtype)
    L = torch.from_numpy(lens).cuda()
    Xd = dev_tensor(X.reshape(cfg.tokens, cfg.d_model), cfg.dtype)
    w = oe.prune_layer(raw, cfg.scheme, cfg.ratio)[0]
    ref = oe.attention_block(X.astype(np.float64), w, cfg.heads, lens, cfg.causal).reshape(cfg.tokens, cfg.d_model)
    whole = etm.attention_fwd(Xd, full, cfg.batch, cfg.seq_len, cfg.heads, L, cfg.causal, ln=False)
    for world in worlds:
        parts = []
        for r in range(world):
            h0, h1 = head_range(cfg.heads, world, r)
            s = pack_head_slice(raw, full, cfg.heads, h0, h1, cfg.dtype)
            p = etm.attention_fwd(Xd, s, cfg.batch, cfg.seq_len, cfg.heads, L, cfg.causal, ln=False,
                                  head_range=(h0, h1))
            assert p.dtype == torch.float32 and p.shape == (cfg.tokens, cfg.d_model)
            parts.append(p)
        total = torch.stack(parts).sum(0)
        torch.cuda.synchronize()
        assert_close(to64(total), ref, what=f"{key} world {world} vs oracle")
        # the same block in one call (FP16/BF16 output): agreement within the storage rounding
        assert_close(to64(total), to64(whole), max_abs=1e-2, rel_fro=2e-3, what=f"{key} world {world} vs full call")


@pytest.mark.parametrize("key,kw,worlds", [
    ("C3", {"layers": 1, "batch": 2}, (2, 3, 8)),
    ("C2", {}, (2, 4)),
    ("C3", {"layers": 1, "batch": 2, "dtype": "bf16"}, (2,)),
    ("C4", {"layers": 1, "batch": 1, "seq_len": 384}, (3,)),
])
def test_head_range_on_full_weights(etm, key, kw, worlds):
    """et_attention_fwd with the FULL packed weights and [head_begin, head_end): the
    library slices W_Q / W_K / W_V by tile rows (a row-pruned W_V is projected whole), runs W_O over a
    full-width Z that is zero outside the range, and folds only the range's pruned-V bias.  The ranks'
    partials sum to the oracle's block and agree with the caller-sliced partials."""
    from paper_conf_sc_chenhplg0d021_b200.dist import head_range, pack_head_slice
    cfg, raws, X, lens = _case(key, **kw)
    raw = raws[0]
    full = etm.pack_layer(raw, cfg.scheme, cfg.ratio, cfg.heads, cfg.dtype)
    L = torch.from_numpy(lens).cuda()
    Xd = dev_tensor(X.reshape(cfg.tokens, cfg.d_model), cfg.dtype)
    w = oe.prune_layer(raw, cfg.scheme, cfg.ratio)[0]
    ref = oe.attention_block(X.astype(np.float64), w, cfg.heads, lens, cfg.causal).reshape(cfg.tokens, cfg.d_model)
    for world in worlds:
        parts = []
        for r in range(world):
            h0, h1 = head_range(cfg.heads, world, r)
            p = etm.attention_fwd(Xd, full, cfg.batch, cfg.seq_len, cfg.heads, L, cfg.causal, ln=False,
                                  head_range=(h0, h1))
            sl = etm.attention_fwd(Xd, pack_head_slice(raw, full, cfg.heads, h0, h1, cfg.dtype), cfg.batch,
                                   cfg.seq_len, cfg.heads, L, cfg.causal, ln=False, head_range=(h0, h1))
            torch.cuda.synchronize()
            assert_close(to64(p), to64(sl), max_abs=2e-3, rel_fro=1e-3, what=f"{key} rank {r}/{world} full vs slices")
            parts.append(p)
        total = torch.stack(parts).sum(0)
        torch.cuda.synchronize()
        assert_close(to64(total), ref, what=f"{key} world {world} (full weights) vs oracle")


def test_head_slice_masks_match_full_pack(etm):
    """The slices keep exactly the full matrices' tiles (bit-exact, unpacked values included)."""
    from paper_conf_sc_chenhplg0d021_b200.dist import pack_head_slice
    cfg, raws, _, _ = _case("C2")
    full = etm.pack_layer(raws[0], cfg.scheme, cfg.ratio, cfg.heads, cfg.dtype)
    dk = cfg.d_k
    s = pack_head_slice(raws[0], full, cfg.heads, 1, 3, cfg.dtype)
    for n in ("wq", "wk", "wv"):
        assert torch.equal(etm.unpack(s.packed[n]), etm.unpack(full.packed[n])[dk:3 * dk])
    assert torch.equal(etm.unpack(s.packed["wo"]), etm.unpack(full.packed["wo"])[:, dk:3 * dk])


def test_head_parallel_rejects_bad_slices(etm):
    from paper_conf_sc_chenhplg0d021_b200.dist import pack_head_slice
    cfg, raws, X, lens = _case("C3", layers=1, batch=1)
    full = etm.pack_layer(raws[0], cfg.scheme, cfg.ratio, cfg.heads, cfg.dtype)
    Xd = dev_tensor(X.reshape(cfg.tokens, cfg.d_model), cfg.dtype)
    s = pack_head_slice(raws[0], full, cfg.heads, 0, 4, cfg.dtype)
    with pytest.raises(etm.EtError):       # slice of 4 heads passed as a 6-head range
        etm.attention_fwd(Xd, s, cfg.batch, cfg.seq_len, cfg.heads, ln=False, head_range=(0, 6),
                          out=torch.empty(cfg.tokens, cfg.d_model, device="cuda"))
    mixed = etm.Layer(dict(full.packed, wo=s.packed["wo"]), full.dense)   # full W_Q/K/V with a sliced W_O
    with pytest.raises(etm.EtError):
        etm.attention_fwd(Xd, mixed, cfg.batch, cfg.seq_len, cfg.heads, ln=False, head_range=(0, 4),
                          out=torch.empty(cfg.tokens, cfg.d_model, device="cuda"))


@pytest.mark.parametrize("world", [2, 3])
def test_head_parallel_encoder_lockstep(etm, world):
    """HeadParallelEncoder on `world` simulated ranks (lock-step on one GPU, partials summed as the
    all-reduce would) equals the float64 oracle encoder; every rank's FFN output is identical."""
    from paper_conf_sc_chenhplg0d021_b200.dist import HeadParallelEncoder
    cfg, raws, X, lens = _case("C3", layers=2, batch=2)
    full = [etm.pack_layer(r, cfg.scheme, cfg.ratio, cfg.heads, cfg.dtype) for r in raws]
    L = torch.from_numpy(lens).cuda()
    encs = [HeadParallelEncoder(raws, full, cfg.heads, cfg.batch, cfg.seq_len, cfg.d_ff, act=cfg.act,
                                ln_eps=cfg.ln_eps, dtype=cfg.dtype, lengths=L, rank=r, world=world)
            for r in range(world)]
    cur = dev_tensor(X.reshape(cfg.tokens, cfg.d_model), cfg.dtype)
    for l in range(cfg.layers):
        total = torch.stack([e.attn_partial(l, cur).clone() for e in encs]).sum(0)
        outs = []
        for e in encs:
            dst = torch.empty_like(cur)
            e.finish_layer(l, cur, total, dst)
            outs.append(dst)
        assert all(torch.equal(o, outs[0]) for o in outs[1:])
        cur = outs[0]
    torch.cuda.synchronize()
    ref = oe.encoder(X.astype(np.float64), [oe.prune_layer(r, cfg.scheme, cfg.ratio)[0] for r in raws], cfg.heads,
                     lens, cfg.causal, cfg.act, cfg.ln_eps).reshape(cfg.tokens, cfg.d_model)
    assert_close(to64(cur), ref, what=f"head-parallel encoder, {world} ranks")


def test_head_parallel_encoder_nccl(etm):
    """The NCCL path end to end (world size 1 on cuda:0: the all-reduce runs through NCCL)."""
    import torch.distributed as dist
    from paper_conf_sc_chenhplg0d021_b200.dist import HeadParallelEncoder
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda:0"))
    try:
        cfg, raws, X, lens = _case("C3", layers=2, batch=2)
        full = [etm.pack_layer(r, cfg.scheme, cfg.ratio, cfg.heads, cfg.dtype) for r in raws]
        L = torch.from_numpy(lens).cuda()
        enc = HeadParallelEncoder(raws, full, cfg.heads, cfg.batch, cfg.seq_len, cfg.d_ff, act=cfg.act,
                                  ln_eps=cfg.ln_eps, dtype=cfg.dtype, lengths=L, rank=0, world=1,
                                  group=dist.group.WORLD)
        Y = enc(dev_tensor(X.reshape(cfg.tokens, cfg.d_model), cfg.dtype))
        torch.cuda.synchronize()
        ref = oe.encoder(X.astype(np.float64), [oe.prune_layer(r, cfg.scheme, cfg.ratio)[0] for r in raws],
                         cfg.heads, lens, cfg.causal, cfg.act, cfg.ln_eps).reshape(cfg.tokens, cfg.d_model)
        assert_close(to64(Y), ref, what="head-parallel encoder over NCCL (world 1)")
    finally:
        dist.destroy_process_group()
