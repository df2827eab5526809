"""Seeded synthetic inputs for MAGIS batched schedule evaluation.

INPUT GENERATION ONLY: graphs shaped like the paper's workloads (Table 2,
P:1751-1760), the F-Trans materialiser (P15), the hot-spot eligible-set
proxy and the counter-based candidate generator.  Both the
CUDA path and the oracle consume these inputs; this package holds none of the
evaluation arithmetic.
"""
from __future__ import annotations

from .graph import Workload, Builder
from .candidates import CandidateGenerator, CandidateSpec, WindowGenerator
from . import models, ftrans, eligible

# SURVEY §8 config sheet.  R_max per config; n_ftrans where applicable.
CONFIGS = {
    "c1": dict(desc="10-op diamond DAGs (brute force)", K=256),
    "c2": dict(desc="ResNet-50 training b64 224^2 fp32", K=65536, R_max=128),
    "c3": dict(desc="BERT-large training s512 b32 fp32, F-Trans n=4 on attention/FFN", K=262144, R_max=256),
    "c4": dict(desc="SD-v1-shaped UNet training b8 1024px bf16, F-Trans n=32 on attention", K=65536, R_max=512),
    "c5": dict(desc="GPT-Neo-1.3B-shaped decoder training s512 b32 bf16", K=1048576, R_max=128),
    # NEXT-4: C3's BERT-large with every attention / FFN group as an F-Trans
    # region offering n in {1, 2, 4} side by side (the candidate picks one)
    "c3f": dict(desc="BERT-large training s512 b32 fp32, F-Trans variant regions n in {1,2,4} per attention/FFN",
                K=65536, R_max=128),
}


def build_workload(cfg: str, **kw) -> Workload:
    """Build the graph of one config (deterministic)."""
    cfg = cfg.lower()
    if cfg == "c1":
        branches = kw.get("branches", [2, 2, 2, 2])
        wl = models.diamond(branches, seed=kw.get("seed", 1))
        return wl
    if cfg == "c2":
        b = models.resnet50(batch=kw.get("batch", 64))
    elif cfg == "c3":
        n = kw.get("ftrans", 4)
        b = models.bert_large(B=kw.get("batch", 32), S=kw.get("seq", 512), ftrans=n)
        b = ftrans.apply(b, n)
    elif cfg == "c4":
        n = kw.get("ftrans", 32)
        b = models.unet_sd(B=kw.get("batch", 8), latent=kw.get("latent", 128), ftrans=n)
        b = ftrans.apply(b, n)
    elif cfg == "c5":
        b = models.gpt_neo_1p3b(B=kw.get("batch", 32), S=kw.get("seq", 512), layers=kw.get("layers", 24))
    elif cfg == "c3f":
        b = models.bert_large(B=kw.get("batch", 32), S=kw.get("seq", 512), ftrans=4,
                              layers=kw.get("layers", 24))
        b = ftrans.apply_variants(b, kw.get("ns", (2, 4)))
    else:
        raise ValueError(cfg)
    wl = b.finish(meta={"config": cfg})
    R_max = kw.get("R_max", CONFIGS[cfg]["R_max"])
    return eligible.select(wl, R_max)


__all__ = ["Workload", "Builder", "CandidateGenerator", "CandidateSpec", "WindowGenerator", "CONFIGS",
           "build_workload", "models", "ftrans", "eligible"]
