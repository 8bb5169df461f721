"""Synthetic training-state workloads C1..C5.

Every tensor carries the parameters of the O9 counter-based generator
(seed, group, gen_id, exponent range, sign rule); both the oracle and the K4
kernel regenerate the same bits from them.  Shapes follow the paper's LLM
workloads (Table 2) scaled to the B200 configs named in
BASELINE.json.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import List, Optional

REQUIRED, OPTIONAL = 0, 1
SEED_BASE = 0x4A4954435F563100  # "JITC_V1\0"

# d.2 value distributions: (lo_exp, hi_exp, force_positive)
KIND_RANGE = {
    "master": (117, 124, False),
    "norm": (126, 127, True),
    "m": (107, 117, False),
    "v": (87, 107, True),
    "grad": (107, 119, False),
    "bytes": (1, 254, False),   # raw-byte test tensors: any finite fp32 pattern
}
DTYPE_CODE = {"u8": 0, "bf16": 1, "f32": 2, "zeros": 3, "ones": 4}
ELEM_BYTES = {"u8": 1, "bf16": 2, "f32": 4, "zeros": 1, "ones": 1}


@dataclass
class TensorSpec:
    name: str
    dtype: str          # "f32" | "bf16" | "u8" | "zeros" | "ones"
    numel: int
    kind: str           # key of KIND_RANGE (ignored for zeros / ones)
    gen_id: int         # tensor_id fed to the generator (a bf16 param uses its master's id)

    @property
    def nbytes(self) -> int:
        return self.numel * ELEM_BYTES[self.dtype]

    @property
    def range(self):
        return KIND_RANGE[self.kind]


@dataclass
class GroupSpec:
    group: int
    policy: int
    members: List[int]
    tensors: List[TensorSpec] = field(default_factory=list)

    @property
    def nbytes(self) -> int:
        return sum(t.nbytes for t in self.tensors)


@dataclass
class Workload:
    name: str
    seed: int
    world: int
    groups: List[GroupSpec]
    chunk_bytes: int = 1 << 20
    note: str = ""

    def groups_of(self, rank: int) -> List[GroupSpec]:
        return [g for g in self.groups if rank in g.members]


# ----------------------------------------------------------------- model shapes
def gpt2_params(n_layer: int, d: int, vocab: int, ctx: int):
    """GPT-2 parameter list [(name, numel, is_norm)] in state-dict order."""
    out = [("wte", vocab * d, False), ("wpe", ctx * d, False)]
    for i in range(n_layer):
        p = f"h.{i}."
        out += [
            (p + "ln_1.weight", d, True), (p + "ln_1.bias", d, False),
            (p + "attn.c_attn.weight", d * 3 * d, False), (p + "attn.c_attn.bias", 3 * d, False),
            (p + "attn.c_proj.weight", d * d, False), (p + "attn.c_proj.bias", d, False),
            (p + "ln_2.weight", d, True), (p + "ln_2.bias", d, False),
            (p + "mlp.c_fc.weight", d * 4 * d, False), (p + "mlp.c_fc.bias", 4 * d, False),
            (p + "mlp.c_proj.weight", 4 * d * d, False), (p + "mlp.c_proj.bias", d, False),
        ]
    out += [("ln_f.weight", d, True), ("ln_f.bias", d, False)]
    return out


def llama_params(n_layer: int, d: int, ffn: int, vocab: int, n_head: int, n_kv: int, tp: int = 1):
    """Llama-3 parameter list for one tensor-parallel shard (Megatron split:
    q/k/v/gate/up column, o/down row, embed/lm_head vocab, norms replicated)."""
    hd = d // n_head
    q, kv = d // tp, n_kv * hd // tp
    out = [("embed_tokens.weight", (vocab // tp) * d, False)]
    for i in range(n_layer):
        p = f"layers.{i}."
        out += [
            (p + "input_layernorm.weight", d, True),
            (p + "self_attn.q_proj.weight", d * q, False),
            (p + "self_attn.k_proj.weight", d * kv, False),
            (p + "self_attn.v_proj.weight", d * kv, False),
            (p + "self_attn.o_proj.weight", q * d, False),
            (p + "post_attention_layernorm.weight", d, True),
            (p + "mlp.gate_proj.weight", d * (ffn // tp), False),
            (p + "mlp.up_proj.weight", d * (ffn // tp), False),
            (p + "mlp.down_proj.weight", (ffn // tp) * d, False),
        ]
    out += [("norm.weight", d, True), ("lm_head.weight", (vocab // tp) * d, False)]
    return out


def _fp32_adam_group(group: int, members, params) -> GroupSpec:
    """C1: fp32 params + Adam m, v, all REQUIRED (12 B/param)."""
    g = GroupSpec(group, REQUIRED, list(members))
    n = len(params)
    for i, (name, numel, is_norm) in enumerate(params):
        g.tensors.append(TensorSpec("param/" + name, "f32", numel, "norm" if is_norm else "master", i))
    for i, (name, numel, _) in enumerate(params):
        g.tensors.append(TensorSpec("exp_avg/" + name, "f32", numel, "m", n + i))
    for i, (name, numel, _) in enumerate(params):
        g.tensors.append(TensorSpec("exp_avg_sq/" + name, "f32", numel, "v", 2 * n + i))
    return g


def _mixed_groups(req: int, opt: int, members, params):
    """bf16 params + fp32 master + m + v (REQUIRED, 14 B/param) and bf16 grads
    (OPTIONAL, 2 B/param): reading R1."""
    n = len(params)
    g = GroupSpec(req, REQUIRED, list(members))
    for i, (name, numel, is_norm) in enumerate(params):   # param = RNE(master): master's id
        g.tensors.append(TensorSpec("param/" + name, "bf16", numel, "norm" if is_norm else "master", n + i))
    for i, (name, numel, is_norm) in enumerate(params):
        g.tensors.append(TensorSpec("master/" + name, "f32", numel, "norm" if is_norm else "master", n + i))
    for i, (name, numel, _) in enumerate(params):
        g.tensors.append(TensorSpec("exp_avg/" + name, "f32", numel, "m", 2 * n + i))
    for i, (name, numel, _) in enumerate(params):
        g.tensors.append(TensorSpec("exp_avg_sq/" + name, "f32", numel, "v", 3 * n + i))
    gr = GroupSpec(opt, OPTIONAL, list(members))
    for i, (name, numel, _) in enumerate(params):
        gr.tensors.append(TensorSpec("grad/" + name, "bf16", numel, "grad", 4 * n + i))
    return g, gr


def c1(world: int = 2) -> Workload:
    p = gpt2_params(4, 256, 3072, 256)
    return Workload("C1-tiny-4M-fp32-adam", SEED_BASE + 1, world,
                    [_fp32_adam_group(0, range(world), p)], note="4,011,520 params; 48,138,240 B")


def c2(world: int = 8) -> Workload:
    p = gpt2_params(48, 1600, 50257, 1024)
    return Workload("C2-gpt2-1.5B", SEED_BASE + 2, world,
                    list(_mixed_groups(0, 1, range(world), p)), note="1,557,611,200 params")


def c3(world: int = 8) -> Workload:
    p = llama_params(32, 4096, 14336, 128256, 32, 8)
    return Workload("C3-llama3-8B", SEED_BASE + 3, world,
                    list(_mixed_groups(0, 1, range(world), p)), note="8,030,261,248 params")


def c4(world: int = 8, shards: int = 4) -> Workload:
    """ZeRO-1: params (bf16, REQUIRED, replicated on all ranks), grads
    (OPTIONAL, replicated), optimizer shard j = flat fp32 master/m/v on ranks
    {j, j+shards, ...} (hybrid when shards < world, pure when shards == world)."""
    p = llama_params(32, 4096, 14336, 128256, 32, 8)
    n = len(p)
    total = sum(x[1] for x in p)
    gp = GroupSpec(0, REQUIRED, list(range(world)))
    gg = GroupSpec(1, OPTIONAL, list(range(world)))
    for i, (name, numel, is_norm) in enumerate(p):
        gp.tensors.append(TensorSpec("param/" + name, "bf16", numel, "norm" if is_norm else "master", i))
        gg.tensors.append(TensorSpec("grad/" + name, "bf16", numel, "grad", n + i))
    groups = [gp, gg]
    per = total // shards
    for j in range(shards):
        gs = GroupSpec(2 + j, REQUIRED, list(range(j, world, shards)))
        gs.tensors = [TensorSpec(f"opt{j}/master", "f32", per, "master", 0),
                      TensorSpec(f"opt{j}/exp_avg", "f32", per, "m", 1),
                      TensorSpec(f"opt{j}/exp_avg_sq", "f32", per, "v", 2)]
        groups.append(gs)
    return Workload(f"C4-zero1-S{shards}", SEED_BASE + 4, world, groups)


def c5(world: int = 8, n_layer: int = 32) -> Workload:
    """Llama-3-70B-shaped TP4 x DP2: group p (REQUIRED) and 4+p (OPTIONAL grads)
    hold TP partition p on ranks {p, p+4}; partitions differ by group id."""
    tp = 4
    p = llama_params(n_layer, 8192, 28672, 128256, 64, 8, tp=tp)
    groups = []
    for part in range(tp):
        g, gr = _mixed_groups(part, tp + part, [part, part + tp], p)
        groups += [g, gr]
    groups.sort(key=lambda g: g.group)
    return Workload("C5-llama3-70B-tp4dp2", SEED_BASE + 5, world, groups)


def scaled(w: Workload, max_numel: int) -> Workload:
    """Same tensor table with every tensor clipped to <= max_numel elements
    (small-but-ragged parity cases; keeps names, dtypes and kinds)."""
    import copy
    w2 = copy.deepcopy(w)
    for g in w2.groups:
        for t in g.tensors:
            t.numel = max(1, min(t.numel, max_numel) - (t.gen_id % 7))
    w2.name += f"-clip{max_numel}"
    return w2


def random_table(seed: int, n: int, max_bytes: int = 4097, group: int = 0) -> GroupSpec:
    """Raw-byte tensors with sizes 1..max_bytes plus all-0x00 / all-0xFF edge
    tensors (SURVEY.md §8(c) c.4, O1/O2/O8 pins)."""
    import random
    r = random.Random(seed)
    g = GroupSpec(group, REQUIRED, [0])
    for i in range(n):
        dt = r.choice(["u8", "u8", "bf16", "f32", "zeros", "ones"])
        eb = ELEM_BYTES[dt]
        numel = max(1, r.randint(1, max_bytes) // eb)
        g.tensors.append(TensorSpec(f"t{i}", dt, numel, "bytes", i))
    return g


CONFIGS = {"C1": c1, "C2": c2, "C3": c3, "C4": c4, "C5": c5}
