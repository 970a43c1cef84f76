"""Tensor-size lists for BASELINE.json's five configs.

Only shapes and sizes live here; no planning or copying.  Every size is in
bytes; names follow the paper's workloads (Bert on PipeDream, GPT on DAPPLE,
P:240-253 Table II).

cfg1  BJ:7   16 fp16 activations x 2,097,152 elements = 4 MiB each, 64 MiB.
cfg2  BJ:8   Bert-large stage 0 (h=1024, 16 heads, FFN 4096, 3 of 24 layers),
             seq 512, micro-batch 8 -> 47 tensors, 900 MiB per micro-batch;
             activation-memory formula 34*s*b*h + 5*a*s^2*b bytes per layer
             (the paper's ref [39]).
cfg3  BJ:9   GPT-10.3B stage 0 fp32 Adam m and v (h=5120, 4 of 32 layers,
             vocab 50257, seq 2048): 100 tensors, 12.21 GB.
cfg4  BJ:10  one uint8 tensor of 4 KiB * 4**k, k = 0..10.
cfg5  BJ:11  sources 0..3 swap (4-s) Bert micro-batch sets (Table IV
             P:347-350: stages 0-3 -> 4-7; memory falls with stage).
"""

KiB = 1024
MiB = 1024 * KiB
GiB = 1024 * MiB

DEFAULT_GRANULE = 64 * KiB


def cfg1_sizes():
    """16 fp16 tensors of 2,097,152 elements (BJ:7)."""
    return [2 * 2_097_152] * 16


def bert_stage0_tensors(seq=512, micro_batch=8, hidden=1024, heads=16,
                        ffn=4096, layers=3):
    """(name, bytes) of Bert stage-0 activations kept for backward, one micro-batch.

    fp16 activations are 2 bytes/element, dropout masks 1 byte/element.
    """
    t = seq * micro_batch                 # tokens
    act = 2 * t * hidden                  # fp16 [T, h]
    mask = t * hidden                     # u8   [T, h]
    att = 2 * heads * seq * seq * micro_batch   # fp16 [b, a, s, s]
    att_mask = heads * seq * seq * micro_batch  # u8
    ffn_act = 2 * t * ffn                 # fp16 [T, 4h]
    out = [("emb_out", act), ("emb_dropout_mask", mask)]
    for l in range(layers):
        out += [
            (f"l{l}.ln1_in", act), (f"l{l}.qkv_in", act), (f"l{l}.q", act),
            (f"l{l}.k", act), (f"l{l}.softmax_out", att),
            (f"l{l}.attn_dropout_mask", att_mask), (f"l{l}.attn_probs", att),
            (f"l{l}.v", act), (f"l{l}.ctx", act),
            (f"l{l}.proj_dropout_mask", mask), (f"l{l}.ln2_in", act),
            (f"l{l}.fc1_in", act), (f"l{l}.gelu_in", ffn_act),
            (f"l{l}.fc2_in", ffn_act), (f"l{l}.fc2_dropout_mask", mask),
        ]
    return out


def cfg2_sizes(micro_batches=1):
    """Bert stage-0 activations for ``micro_batches`` in-flight micro-batches."""
    one = [b for _, b in bert_stage0_tensors()]
    return one * micro_batches


def gpt_stage0_params(hidden=5120, layers=4, vocab=50257, seq=2048):
    """(name, elements) of GPT stage-0 parameters (4 of 32 layers + embeddings)."""
    h = hidden
    out = [("tok_emb", vocab * h), ("pos_emb", seq * h)]
    for l in range(layers):
        out += [
            (f"l{l}.ln1_w", h), (f"l{l}.ln1_b", h),
            (f"l{l}.qkv_w", 3 * h * h), (f"l{l}.qkv_b", 3 * h),
            (f"l{l}.proj_w", h * h), (f"l{l}.proj_b", h),
            (f"l{l}.ln2_w", h), (f"l{l}.ln2_b", h),
            (f"l{l}.fc1_w", 4 * h * h), (f"l{l}.fc1_b", 4 * h),
            (f"l{l}.fc2_w", 4 * h * h), (f"l{l}.fc2_b", h),
        ]
    return out


def cfg3_tensors():
    """(name, bytes) of fp32 Adam m and v for every stage-0 parameter."""
    out = []
    for name, n in gpt_stage0_params():
        out.append((name + ".adam_m", 4 * n))
        out.append((name + ".adam_v", 4 * n))
    return out


def cfg3_sizes():
    return [b for _, b in cfg3_tensors()]


def cfg4_sizes():
    """4 KiB * 4**k for k = 0..10 (4 KiB .. 4 GiB)."""
    return [4 * KiB * 4 ** k for k in range(11)]


def cfg5_source_sizes(source):
    """Source s in 0..3 swaps (4-s) Bert micro-batch sets."""
    assert 0 <= source <= 3
    return cfg2_sizes(micro_batches=4 - source)


# Topologies: (world, source, peers, spare bytes per peer) per config.
CONFIGS = {
    1: dict(world=2, source=0, peers=[1], spare=1 * GiB),
    2: dict(world=4, source=0, peers=[1, 2, 3], spare=24 * GiB),
    3: dict(world=8, source=0, peers=[5, 6, 7],
            spare_by_peer={5: 8 * GiB, 6: 8 * GiB, 7: 2 * GiB}),
    4: dict(sweeps=[(2, 1), (4, 3), (8, 7), (8, 1), (8, 3)], spare=8 * GiB),
    5: dict(world=8, sources=[0, 1, 2, 3], peers=[4, 5, 6, 7], spare=16 * GiB),
}


def spare_vector(world, source, peers, spare=None, spare_by_peer=None):
    """Per-device spare bytes: ``spare`` on each listed peer, 0 elsewhere."""
    v = [0] * world
    for p in peers:
        v[p] = spare_by_peer[p] if spare_by_peer is not None else spare
    return v


def bw_vector(world, source, peers, weight=1):
    """Equal NVSwitch link weights to the listed peers (R10), 0 elsewhere."""
    v = [0] * world
    for p in peers:
        v[p] = weight
    return v
