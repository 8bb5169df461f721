"""Synthetic training state on the GPU for tests and bench (harness, not the
method): allocates one device arena per group, places the tensors in a
shuffled order at 512-byte alignment (like PyTorch's caching allocator), and
fills them with the K4 counter-based generator (jitc_gen_fill)."""
from __future__ import annotations

import random
from typing import List, Tuple

import torch

from workloads.configs import DTYPE_CODE, ELEM_BYTES, GroupSpec, TensorSpec

from . import jitc


class GroupState:
    def __init__(self, g: GroupSpec, seed: int, device: int = 0, align: int = 512, misalign: int = 0,
                 shuffle_seed: int = 1, fill: bool = True):
        self.spec, self.seed = g, seed
        sizes = [t.nbytes for t in g.tensors]
        order = list(range(len(sizes)))
        random.Random(shuffle_seed).shuffle(order)
        offs = [0] * len(sizes)
        pos = 0
        for i in order:
            # misaligned placement (tests): shift every third tensor by `misalign`
            # bytes, rounded up to its element size (an fp32 tensor is never
            # less than 4-byte aligned in a real program)
            eb = ELEM_BYTES[g.tensors[i].dtype]
            shift = 0 if not (misalign and i % 3 == 1) else (misalign if misalign % eb == 0 else eb)
            offs[i] = pos + shift
            pos = (offs[i] + sizes[i] + align - 1) // align * align
        self.arena = torch.empty(max(pos, 1), dtype=torch.uint8, device=f"cuda:{device}")
        base = self.arena.data_ptr()
        self.ptrs = [base + o for o in offs]
        self.offs = offs
        if fill:
            self.fill()

    def fill(self, stream: int = 0):
        for t, p in zip(self.spec.tensors, self.ptrs):
            lo, hi, pos = t.range
            jitc.gen_fill(p, DTYPE_CODE[t.dtype], t.numel, self.seed, self.spec.group, t.gen_id, lo, hi, pos, stream)
        # the library works on its own non-blocking streams: finish the writes first
        torch.cuda.current_stream().synchronize() if not stream else torch.cuda.ExternalStream(stream).synchronize()

    def table(self) -> List[Tuple[str, int, int, int]]:
        return [(t.name, p, t.nbytes, DTYPE_CODE[t.dtype]) for t, p in zip(self.spec.tensors, self.ptrs)]

    def tensor_bytes(self, i: int) -> torch.Tensor:
        o, n = self.offs[i], self.spec.tensors[i].nbytes
        return self.arena[o:o + n]

    @property
    def nbytes(self) -> int:
        return sum(t.nbytes for t in self.spec.tensors)

    def scramble(self):
        """Overwrite every tensor (a replacement rank's uninitialised memory)."""
        self.arena.fill_(0xA5)
        torch.cuda.current_stream().synchronize()
