"""PyTorch integration of the phase word (A2): the pre- and post-optimizer-step
hooks of PAPER.md:188 ("pre-optimizer-step and post-optimizer-step callback
hooks in the ML framework such as PyTorch, which inform [the library] about
the start and end of the optimizer step").

    ctx = J.Context(...)
    table = state_table(model, optimizer)               # names from the state dict
    ctx.register(0, J.REQUIRED, members, table, keepalive=(model, optimizer))
    attach(ctx, optimizer, group=0)                      # DIRTY before step(), v+1 after

Both hooks only enqueue jitc_mark on the current CUDA stream (one 8-byte
cuStreamWriteValue64 into mapped host memory, ordered after the optimizer
kernels already queued there): no kernel, no synchronisation, so the
steady-state overhead stays at the paper's "no measurable increase"
(Table 4).  Argument marshalling only -- the library does
the work.
"""
from __future__ import annotations

from typing import List, Optional, Tuple

import torch

from . import jitc as J

DT = {torch.uint8: 0, torch.bfloat16: 1, torch.float32: 2}


def _dtype(t: torch.Tensor) -> int:
    return DT.get(t.dtype, 100 + t.element_size())


def state_table(model: torch.nn.Module, optimizer: Optional[torch.optim.Optimizer] = None,
                grads: bool = False) -> List[Tuple[str, int, int, int]]:
    """[(name, device_ptr, nbytes, dtype)] of the parameters and, for Adam /
    AdamW, the exp_avg / exp_avg_sq / step state -- the training state the
    paper checkpoints.  Names are state-dict keys, identical on
    every replica (reading R5).  The optimizer state must exist (after the
    first step, or torch's _init_group)."""
    out = []
    names = {p: n for n, p in model.named_parameters()}
    for n, p in model.named_parameters():
        if not p.is_cuda or not p.is_contiguous():
            raise ValueError(f"{n}: only contiguous CUDA tensors can be registered")
        out.append(("param/" + n, p.data_ptr(), p.numel() * p.element_size(), _dtype(p)))
    if optimizer is not None:
        for group in optimizer.param_groups:
            for p in group["params"]:
                st = optimizer.state.get(p, {})
                for key in sorted(st):
                    v = st[key]
                    if isinstance(v, torch.Tensor) and v.is_cuda:
                        out.append((f"{key}/{names[p]}", v.data_ptr(), v.numel() * v.element_size(), _dtype(v)))
    if grads:
        for n, p in model.named_parameters():
            if p.grad is not None:
                out.append(("grad/" + n, p.grad.data_ptr(), p.grad.numel() * p.grad.element_size(), _dtype(p.grad)))
    return out


class Hooks:
    def __init__(self, handles, counter):
        self.handles = handles
        self.counter = counter

    @property
    def version(self) -> int:
        return self.counter[0]

    def remove(self):
        for h in self.handles:
            h.remove()


def attach(ctx: "J.Context", optimizer: torch.optim.Optimizer, group: int, version: int = 0) -> Hooks:
    """Registers the optimizer pre/post step hooks: mark(group, v, DIRTY)
    before step(), mark(group, v+1, CLEAN) after it, on the current stream."""
    counter = [version]
    ctx.mark(group, version, J.CLEAN)

    def pre(opt, args, kwargs):
        ctx.mark(group, counter[0], J.DIRTY, torch.cuda.current_stream().cuda_stream)

    def post(opt, args, kwargs):
        counter[0] += 1
        ctx.mark(group, counter[0], J.CLEAN, torch.cuda.current_stream().cuda_stream)

    return Hooks([optimizer.register_step_pre_hook(pre), optimizer.register_step_post_hook(post)], counter)
