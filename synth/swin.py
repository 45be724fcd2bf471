"""Seeded Swin-Transformer inputs, weights and model constants (Table 2: Swin-B).

Holds NO arithmetic of Souffle's method.  Besides seeded draws it builds the two constant tensors
that are part of the Swin model definition (Liu et al. 2021, torchvision `swin_b`) and that a TE
program consumes as plain inputs, like weights:
  * the dense relative-position bias [heads, w*w, w*w], gathered from the learned table
    [(2w-1)^2, heads] by the fixed relative-position index (a data-dependent gather is not an
    affine TE, reading R15; done once at weight-preparation time like the embedding
    gather of BERT);
  * the shifted-window attention mask [nW, 1, w*w, w*w] (0 inside a region, -100 across regions).
Both are pinned by the oracle test against torchvision's own implementation.

Recipe: image ~ N(0,1) [B, 3, 224, 224] fp32; GEMM weights ~ N(0, 1/K)
stored [N, K] in the config's GEMM dtype; biases N(0, 0.02^2); LN gamma = 1 + N(0, 0.1^2),
beta = N(0, 0.1^2); relative-position table N(0, 0.5^2).  Seeds: input 1234; block weights
1000 * (global block index + 1) + slot; patch embedding 1..4; patch merge i 500000 + 10 i + slot;
head 900000 + slot.
"""
from __future__ import annotations

import numpy as np

from . import INPUT_SEED, normal

# torchvision swin_b (Table 2: 224 x 224, window 7)
SWIN_B = dict(name="swin_b", image=224, patch=4, embed=128, depths=(2, 2, 18, 2), heads=(4, 8, 16, 32),
              window=7, mlp_ratio=4, classes=1000, eps=1e-5, gemm_dtype="bf16", batch=1)
# parity config: both stages of the structure (a shifted stage, a patch merge, an unshifted stage
# whose window covers the whole map) at a size the fp64 oracle runs in well under a second
SWIN_TINY = dict(name="swin_tiny", image=56, patch=4, embed=32, depths=(2, 2), heads=(2, 4), window=7,
                 mlp_ratio=4, classes=10, eps=1e-5, gemm_dtype="f32", batch=1)

BLOCK_SLOTS = dict(g1=1, be1=2, Wqkv=3, bqkv=4, table=5, Wproj=6, bproj=7, g2=8, be2=9, W1=10, b1=11, W2=12, b2=13)


def stage_res(cfg, i):
    return cfg["image"] // cfg["patch"] // (2 ** i)


def shift_of(cfg, i, j):
    """torchvision: odd blocks shift by w//2, unless the window covers the whole feature map."""
    w = cfg["window"]
    if j % 2 == 0 or w >= stage_res(cfg, i):
        return 0
    return w // 2


def relative_position_index(w: int) -> np.ndarray:
    """[w*w, w*w] index into the (2w-1)^2 table (the fixed gather of the Swin model)."""
    c = np.stack(np.meshgrid(np.arange(w), np.arange(w), indexing="ij")).reshape(2, -1)
    rel = (c[:, :, None] - c[:, None, :]).transpose(1, 2, 0)
    rel[:, :, 0] += w - 1
    rel[:, :, 1] += w - 1
    rel[:, :, 0] *= 2 * w - 1
    return rel.sum(-1)


def dense_bias(table: np.ndarray, w: int) -> np.ndarray:
    """table [(2w-1)^2, heads] -> [heads, w*w, w*w] fp32."""
    idx = relative_position_index(w)
    return np.ascontiguousarray(table[idx.reshape(-1)].reshape(w * w, w * w, -1).transpose(2, 0, 1)).astype(np.float32)


def shift_mask(res: int, w: int, s: int) -> np.ndarray:
    """[nW, 1, w*w, w*w] additive mask of shifted-window attention (0 / -100)."""
    region = np.zeros((res, res), dtype=np.int64)
    cnt = 0
    for hs in (slice(0, res - w), slice(res - w, res - s), slice(res - s, res)):
        for ws in (slice(0, res - w), slice(res - w, res - s), slice(res - s, res)):
            region[hs, ws] = cnt
            cnt += 1
    n = res // w
    win = region.reshape(n, w, n, w).transpose(0, 2, 1, 3).reshape(n * n, w * w)
    diff = win[:, None, :] - win[:, :, None]
    return np.where(diff != 0, -100.0, 0.0).astype(np.float32)[:, None, :, :]


def _block_params(cfg, gb, C, nh):
    wd = cfg["gemm_dtype"]
    s = lambda k: 1000 * (gb + 1) + BLOCK_SLOTS[k]
    w = lambda k, shp: normal(s(k), shp, std=1.0 / np.sqrt(shp[1]), dtype=wd)
    v = lambda k, shp: normal(s(k), shp, std=0.02)
    F = cfg["mlp_ratio"] * C
    win = cfg["window"]
    return dict(g1=normal(s("g1"), (C,), std=0.1, mean=1.0), be1=normal(s("be1"), (C,), std=0.1),
                Wqkv=w("Wqkv", (3 * C, C)), bqkv=v("bqkv", (3 * C,)),
                table=normal(s("table"), ((2 * win - 1) ** 2, nh), std=0.5),
                Wproj=w("Wproj", (C, C)), bproj=v("bproj", (C,)),
                g2=normal(s("g2"), (C,), std=0.1, mean=1.0), be2=normal(s("be2"), (C,), std=0.1),
                W1=w("W1", (F, C)), b1=v("b1", (F,)), W2=w("W2", (C, F)), b2=v("b2", (C,)))


def swin_params(cfg: dict) -> dict:
    """Every learned parameter (torchvision layout; conv weight flattened to [C, 3*p*p])."""
    C, p, wd = cfg["embed"], cfg["patch"], cfg["gemm_dtype"]
    P = dict(Wpe=normal(1, (C, 3 * p * p), std=1.0 / np.sqrt(3 * p * p), dtype=wd), bpe=normal(2, (C,), std=0.02),
             gpe=normal(3, (C,), std=0.1, mean=1.0), bepe=normal(4, (C,), std=0.1), blocks=[], merges=[])
    gb = 0
    for i, (depth, nh) in enumerate(zip(cfg["depths"], cfg["heads"])):
        for j in range(depth):
            P["blocks"].append(_block_params(cfg, gb, C, nh))
            gb += 1
        if i < len(cfg["depths"]) - 1:
            base = 500000 + 10 * i
            P["merges"].append(dict(g=normal(base + 1, (4 * C,), std=0.1, mean=1.0),
                                    be=normal(base + 2, (4 * C,), std=0.1),
                                    W=normal(base + 3, (2 * C, 4 * C), std=1.0 / np.sqrt(4 * C), dtype=wd)))
            C *= 2
    P["gn"] = normal(900001, (C,), std=0.1, mean=1.0)
    P["ben"] = normal(900002, (C,), std=0.1)
    P["Wh"] = normal(900003, (cfg["classes"], C), std=1.0 / np.sqrt(C), dtype=wd)
    P["bh"] = normal(900004, (cfg["classes"],), std=0.02)
    return P


def swin_input(cfg: dict, seed: int = INPUT_SEED) -> np.ndarray:
    return normal(seed, (cfg["batch"], 3, cfg["image"], cfg["image"]))


def swin_feed_values(cfg: dict, P: dict) -> dict:
    """Name -> value of every placeholder the Swin TE program takes, in the names both builders use:
    learned parameters plus the model constants (dense relative-position bias, shift masks)."""
    out = {"Wpe": P["Wpe"], "bpe": P["bpe"], "gpe": P["gpe"], "bepe": P["bepe"], "gn": P["gn"], "ben": P["ben"],
           "Wh": P["Wh"], "bh": P["bh"]}
    gb = 0
    for i, depth in enumerate(cfg["depths"]):
        R = stage_res(cfg, i)
        for j in range(depth):
            bp = P["blocks"][gb]
            for k, v in bp.items():
                if k != "table":
                    out[f"b{gb}.{k}"] = v
            out[f"b{gb}.bias"] = dense_bias(bp["table"], cfg["window"])
            s = shift_of(cfg, i, j)
            if s:
                out[f"b{gb}.mask"] = shift_mask(R, cfg["window"], s)
            gb += 1
        if i < len(cfg["depths"]) - 1:
            for k, v in P["merges"][i].items():
                out[f"m{i}.{k}"] = v
    return out
