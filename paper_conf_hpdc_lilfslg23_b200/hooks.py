"""PyTorch activation detector: the SRU case —
NaN from an uninitialised tensor caught downstream — recast for model code.

Forward hooks scan every module output with ``fpx_scan_tensor`` (one launch
per output, on the current stream, never synchronising), site = the module's
index in ``model.named_modules()`` order.  Every scanned output gets its own
index range in execution order: ``first_index = seq << 36 | element`` where
``seq`` counts scans, so the entry with the smallest first_index is the first
output (in execution order) holding an exceptional value;
``first_exception()`` resolves it to (forward call, module, element, kind).
"""
from __future__ import annotations

import torch

from . import fpx

SEQ_SHIFT = 36  # element indices below 2^36 per scanned output


class SelectivePolicy:
    """Alg3, selective instrumentation, at the API level: scan a
    kernel / module only if it is in the white-list (when one is given) and
    only on one in every k of its invocations (freq-redn-factor; k = 0 or 1:
    every invocation).  ``num[name]`` counts invocations as in Alg3 line 14."""

    def __init__(self, white_list=None, k: int = 0):
        self.white = set(white_list) if white_list else None
        self.k = k
        self.num = {}

    def should_scan(self, name: str) -> bool:
        instr = self.white is None or name in self.white      # Alg3 lines 2-9
        n = self.num.get(name, 0)
        if self.k not in (0, 1) and n % self.k != 0:          # Alg3 lines 10-13
            instr = False
        self.num[name] = n + 1                                # Alg3 line 14
        return instr


class ActivationScanner:
    def __init__(self, model: torch.nn.Module, handle: "fpx.Handle | None" = None, leaf_only: bool = True,
                 device: int | None = None, policy: SelectivePolicy | None = None, batch: bool = False):
        """batch=True: collect every output of a forward call and scan them all
        with ONE fused launch (fpx_scan_tensors) when the call returns."""
        self.model = model
        self.policy = policy
        self.batch = batch
        self._queue = []
        dev = torch.cuda.current_device() if device is None else device
        self.handle = handle if handle is not None else fpx.Handle(dev)
        self._own = handle is None
        self.names = []
        self._hooks = []
        self.calls = 0
        self.seq = []  # seq -> (forward call, site)
        for name, mod in model.named_modules():
            if leaf_only and any(True for _ in mod.children()):
                continue
            site = len(self.names)
            self.names.append(name or "<root>")
            self._hooks.append(mod.register_forward_hook(self._make_hook(site)))
        self._pre = model.register_forward_pre_hook(self._on_call)
        self._post = model.register_forward_hook(self._on_return) if batch else None

    def _on_call(self, module, args):
        self.calls += 1

    def _on_return(self, module, args, out):
        if self._queue:
            self.handle.scan_tensors(self._queue)
            self._queue = []

    def _make_hook(self, site: int):
        def hook(module, args, out):
            if self.policy is None or self.policy.should_scan(self.names[site]):
                self._scan(out, site)

        return hook

    def _scan(self, out, site: int):
        if isinstance(out, torch.Tensor):
            if out.is_cuda and out.dtype in (torch.float32, torch.float64, torch.float16, torch.bfloat16):
                t = out if out.is_contiguous() else out.contiguous()
                assert t.numel() < (1 << SEQ_SHIFT)
                base = len(self.seq) << SEQ_SHIFT
                if self.batch:
                    self._queue.append((t, site, base))
                else:
                    self.handle.scan_tensor(t, site=site, base_index=base)
                self.seq.append((self.calls, site))
        elif isinstance(out, (tuple, list)):
            for o in out:
                self._scan(o, site)
        elif isinstance(out, dict):
            for o in out.values():
                self._scan(o, site)

    def entries(self):
        return self.handle.fetch()

    def first_exception(self, kinds=(fpx.NAN, fpx.INF)):
        """(call, module name, element, kind) of the earliest exceptional value
        of the given kinds, or None."""
        ents = self.entries()
        ents = ents[[int(k) in kinds for k in ents["kind"]]] if len(ents) else ents
        if len(ents) == 0:
            return None
        e = ents[int(ents["first_index"].argmin())]
        fi = int(e["first_index"])
        call, site = self.seq[fi >> SEQ_SHIFT]
        return call, self.names[site], fi & ((1 << SEQ_SHIFT) - 1), int(e["kind"])

    def remove(self):
        for h in self._hooks:
            h.remove()
        self._pre.remove()
        if self._post is not None:
            self._post.remove()
        self._hooks = []
        if self._own:
            self.handle.close()
