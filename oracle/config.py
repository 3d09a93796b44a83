"""Model shapes and the canonical tensor enumeration (oracle side).

Shapes: public FLUX.1-dev (S:§8(c) S1; BASELINE.json configs: hidden 3072,
24 heads, 19 double + 38 single blocks) and the "tiny" block of config 1
(hidden 256, 4 heads, 1 double block; L_i = 256, L_t = 64).

Tensor ids (restated independently in include/tsv.h, "Tensor ids"):
  global   0 img_in.w [h,in]   1 img_in.b [h]    2 txt_in.w [h,ctx]  3 txt_in.b [h]
           4 time_in.in.w [h,256] 5 .b  6 time_in.out.w [h,h] 7 .b
           8 guidance_in.in.w [h,256] 9 .b 10 guidance_in.out.w [h,h] 11 .b
          12 vector_in.in.w [h,vec] 13 .b 14 vector_in.out.w [h,h] 15 .b
          16 final.mod.w [2h,h] 17 final.mod.b [2h] 18 final.lin.w [in,h] 19 final.lin.b [in]
  double j, stream s (0 = img, 1 = txt): base 64 + 32 j + 16 s
          +0 mod.w [6h,h] +1 mod.b [6h] +2 qkv.w [3h,h] +3 qkv.b [3h]
          +4 q_norm.g [D] +5 k_norm.g [D] +6 proj.w [h,h] +7 proj.b [h]
          +8 fc1.w [F,h] +9 fc1.b [F] +10 fc2.w [h,F] +11 fc2.b [h]
  single j: base 4096 + 16 j
          +0 mod.w [3h,h] +1 mod.b [3h] +2 lin1.w [3h+F,h] +3 lin1.b [3h+F]
          +4 q_norm.g [D] +5 k_norm.g [D] +6 lin2.w [h,h+F] +7 lin2.b [h]
  request inputs (seed = request seed): 1 x_T [L_i,in] (fp32) 2 T [L_t,ctx] 3 y [vec]

SD3-medium family (S:§8(c) O-SD3; family == "sd3"): the same ids where the tensor
exists.  Globals 0-7, 12-19 (no guidance embedder; img_in = the 2x2 patch-embed conv
flattened in (c, ph, pw) order; final.mod rows are (scale, shift), S7).  Joint block j,
stream s (0 = img, 1 = txt) uses the double-block ids above minus the QK-norm gains
(+4, +5); qkv.w stacks to_q; to_k; to_v (img) or add_q; add_k; add_v (txt).  The txt
stream of the last block is context_pre_only: +0 mod.w [2h,h] (scale, shift), +1 mod.b
[2h], +2 qkv.w, +3 qkv.b only.  Request inputs: 1 x_T, 2 T_c, 3 y_c (conditional),
4 T_u [L_t,ctx], 5 y_u [vec] (unconditional, CFG batch 2, S23).
"""
from __future__ import annotations

from dataclasses import dataclass, field

WEIGHT_SEED = 0x7E7125E7  # S:§8(d) "weight_seed = 0x7E7125E7"


@dataclass(frozen=True)
class ModelCfg:
    name: str
    hidden: int
    heads: int
    head_dim: int
    mlp_hidden: int
    n_double: int
    n_single: int
    in_ch: int = 64
    ctx_dim: int = 4096
    vec_dim: int = 768
    text_tokens: int = 512
    axes_dim: tuple = (16, 56, 56)
    theta: float = 10000.0
    guidance_embed: bool = True
    family: str = "flux"
    cfg_scale: float = 7.0      # SD3 classifier-free guidance scale (S:§8(c) O-SD3)
    shift: float = 3.0          # SD3 flow-matching schedule shift
    pe_max: int = 192           # SD3 pos_embed_max_size
    pe_base: int = 64           # SD3 base_size = sample_size / patch_size


FLUX = ModelCfg("flux", 3072, 24, 128, 12288, 19, 38)
TINY = ModelCfg("tiny", 256, 4, 64, 1024, 1, 0, in_ch=64, ctx_dim=512, vec_dim=256,
                text_tokens=64, axes_dim=(8, 28, 28))
TINY_S = ModelCfg("tiny_s", 256, 4, 64, 1024, 1, 1, in_ch=64, ctx_dim=512, vec_dim=256,
                  text_tokens=64, axes_dim=(8, 28, 28))
TINY2 = ModelCfg("tiny2", 256, 4, 64, 1024, 2, 2, in_ch=64, ctx_dim=512, vec_dim=256,
                 text_tokens=64, axes_dim=(8, 28, 28))
SD3 = ModelCfg("sd3", 1536, 24, 64, 6144, 24, 0, in_ch=64, ctx_dim=4096, vec_dim=2048, text_tokens=333,
               axes_dim=(), guidance_embed=False, family="sd3")
TINY_SD3 = ModelCfg("tiny_sd3", 256, 4, 64, 1024, 2, 0, in_ch=64, ctx_dim=512, vec_dim=256, text_tokens=77,
                    axes_dim=(), guidance_embed=False, family="sd3")
MODELS = {m.name: m for m in (FLUX, TINY, TINY_S, TINY2, SD3, TINY_SD3)}


def double_base(j: int, s: int) -> int:
    return 64 + 32 * j + 16 * s


def single_base(j: int) -> int:
    return 4096 + 16 * j


def tensor_table(cfg: ModelCfg):
    """List of (tensor_id, name, shape, kind, fan_in)."""
    if cfg.family == "sd3":
        return sd3_tensor_table(cfg)
    h, D, F, i = cfg.hidden, cfg.head_dim, cfg.mlp_hidden, cfg.in_ch
    t = [
        (0, "img_in.w", (h, i), "w", i), (1, "img_in.b", (h,), "b", None),
        (2, "txt_in.w", (h, cfg.ctx_dim), "w", cfg.ctx_dim), (3, "txt_in.b", (h,), "b", None),
        (4, "time_in.in.w", (h, 256), "w", 256), (5, "time_in.in.b", (h,), "b", None),
        (6, "time_in.out.w", (h, h), "w", h), (7, "time_in.out.b", (h,), "b", None),
        (8, "guidance_in.in.w", (h, 256), "w", 256), (9, "guidance_in.in.b", (h,), "b", None),
        (10, "guidance_in.out.w", (h, h), "w", h), (11, "guidance_in.out.b", (h,), "b", None),
        (12, "vector_in.in.w", (h, cfg.vec_dim), "w", cfg.vec_dim), (13, "vector_in.in.b", (h,), "b", None),
        (14, "vector_in.out.w", (h, h), "w", h), (15, "vector_in.out.b", (h,), "b", None),
        (16, "final.mod.w", (2 * h, h), "w", h), (17, "final.mod.b", (2 * h,), "b", None),
        (18, "final.lin.w", (i, h), "w", h), (19, "final.lin.b", (i,), "b", None),
    ]
    for j in range(cfg.n_double):
        for s, sn in ((0, "img"), (1, "txt")):
            b = double_base(j, s)
            p = f"double{j}.{sn}."
            t += [
                (b + 0, p + "mod.w", (6 * h, h), "w", h), (b + 1, p + "mod.b", (6 * h,), "b", None),
                (b + 2, p + "qkv.w", (3 * h, h), "w", h), (b + 3, p + "qkv.b", (3 * h,), "b", None),
                (b + 4, p + "q_norm.g", (D,), "g", None), (b + 5, p + "k_norm.g", (D,), "g", None),
                (b + 6, p + "proj.w", (h, h), "w", h), (b + 7, p + "proj.b", (h,), "b", None),
                (b + 8, p + "fc1.w", (F, h), "w", h), (b + 9, p + "fc1.b", (F,), "b", None),
                (b + 10, p + "fc2.w", (h, F), "w", F), (b + 11, p + "fc2.b", (h,), "b", None),
            ]
    for j in range(cfg.n_single):
        b = single_base(j)
        p = f"single{j}."
        t += [
            (b + 0, p + "mod.w", (3 * h, h), "w", h), (b + 1, p + "mod.b", (3 * h,), "b", None),
            (b + 2, p + "lin1.w", (3 * h + F, h), "w", h), (b + 3, p + "lin1.b", (3 * h + F,), "b", None),
            (b + 4, p + "q_norm.g", (D,), "g", None), (b + 5, p + "k_norm.g", (D,), "g", None),
            (b + 6, p + "lin2.w", (h, h + F), "w", h + F), (b + 7, p + "lin2.b", (h,), "b", None),
        ]
    return t


def sd3_tensor_table(cfg: ModelCfg):
    """SD3-medium (diffusers SD3Transformer2DModel names in comments): see the module header."""
    h, F, i = cfg.hidden, cfg.mlp_hidden, cfg.in_ch
    t = [
        (0, "img_in.w", (h, i), "w", i), (1, "img_in.b", (h,), "b", None),          # pos_embed.proj
        (2, "txt_in.w", (h, cfg.ctx_dim), "w", cfg.ctx_dim), (3, "txt_in.b", (h,), "b", None),  # context_embedder
        (4, "time_in.in.w", (h, 256), "w", 256), (5, "time_in.in.b", (h,), "b", None),  # timestep_embedder
        (6, "time_in.out.w", (h, h), "w", h), (7, "time_in.out.b", (h,), "b", None),
        (12, "vector_in.in.w", (h, cfg.vec_dim), "w", cfg.vec_dim), (13, "vector_in.in.b", (h,), "b", None),
        (14, "vector_in.out.w", (h, h), "w", h), (15, "vector_in.out.b", (h,), "b", None),  # text_embedder
        (16, "final.mod.w", (2 * h, h), "w", h), (17, "final.mod.b", (2 * h,), "b", None),  # norm_out
        (18, "final.lin.w", (i, h), "w", h), (19, "final.lin.b", (i,), "b", None),          # proj_out
    ]
    for j in range(cfg.n_double):
        for s, sn in ((0, "img"), (1, "txt")):
            b = double_base(j, s)
            p = f"joint{j}.{sn}."
            if s == 1 and j == cfg.n_double - 1:    # context_pre_only
                t += [(b + 0, p + "mod.w", (2 * h, h), "w", h), (b + 1, p + "mod.b", (2 * h,), "b", None),
                      (b + 2, p + "qkv.w", (3 * h, h), "w", h), (b + 3, p + "qkv.b", (3 * h,), "b", None)]
                continue
            t += [
                (b + 0, p + "mod.w", (6 * h, h), "w", h), (b + 1, p + "mod.b", (6 * h,), "b", None),
                (b + 2, p + "qkv.w", (3 * h, h), "w", h), (b + 3, p + "qkv.b", (3 * h,), "b", None),
                (b + 6, p + "proj.w", (h, h), "w", h), (b + 7, p + "proj.b", (h,), "b", None),
                (b + 8, p + "fc1.w", (F, h), "w", h), (b + 9, p + "fc1.b", (F,), "b", None),
                (b + 10, p + "fc2.w", (h, F), "w", F), (b + 11, p + "fc2.b", (h,), "b", None),
            ]
    return t


def image_tokens(height_px: int, width_px: int) -> int:
    """L_i = (H/16)(W/16): 8x VAE downsampling then 2x2 patching (Table 1)."""
    if height_px % 16 or width_px % 16:
        raise ValueError("height and width must be multiples of 16")
    return (height_px // 16) * (width_px // 16)


@dataclass
class Request:
    height: int
    width: int
    num_steps: int = 20
    seed: int = 1000
    guidance: float = 3.5
    extra: dict = field(default_factory=dict)
