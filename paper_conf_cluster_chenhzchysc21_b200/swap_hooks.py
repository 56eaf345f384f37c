"""Training integration: the swapping executor of PAPER.md Fig. 4
(:108) and §IV-A (:118-120) attached to autograd.  Every activation an op saves for backward
(ReLU / MaxPool outputs = the inputs of the next conv) is swapped out to
pinned host memory through libcswap when it is saved, and swapped back in when backward needs it,
with the next one prefetched while the current backward layer runs (Fig. 2, :64-:72: Prefetch_n
overlaps B_{n+1}).

Policies (§V, :251):
  "resident"  no swapping (all activations stay in HBM);
  "none"      vDNN: offload every candidate uncompressed (:70-72);
  "zvc"       SC: always ZVC (:80-82);
  "auto"      CSWAP: per tensor, sparsity probe + cost model (Eq. 1-4, :137-154) with the tensor's
              hidden latencies Hidden_f / Hidden_b (Table II, :129-130) measured by `profile()`;
  an int      force one codec id (tests).

The tensor profiler (A1): `profile(step_fn)` runs one step with CUDA events at
every save (forward) and every use (backward) of a candidate; Hidden_f(i) is the forward time
from saving tensor i to saving tensor i+1 (the compute its offload can overlap) and Hidden_b(i)
the backward time from using tensor i+1 to using tensor i (the compute its prefetch can overlap).

Only argument marshalling and bookkeeping live here; every byte is moved and (de)compressed by
libcswap's kernels.
"""
from __future__ import annotations

import dataclasses
import weakref

import torch

from . import cswap as C

_DTYPES = {torch.float32: C.F32, torch.float16: C.F16, torch.bfloat16: C.BF16}
POLICIES = {"none": C.NONE, "zvc": C.ZVC, "auto": C.AUTO}


class CSwapBackend:
    """Moves tensors through libcswap (the product path)."""

    def __init__(self, device: int | None = None):
        dev = torch.cuda.current_device() if device is None else device
        C.init(dev)
        self.keep = torch.cuda.Stream(dev)      # waits for raw offloads (keeps d_in alive)
        self.prefetch = torch.cuda.Stream(dev)  # swap-in of the next tensor during backward

    @staticmethod
    def accepts(t: torch.Tensor) -> bool:
        return t.is_cuda

    def swap_out(self, t: torch.Tensor, codec: int, hidden_f: float, hidden_b: float):
        flat = t.reshape(-1)
        h = C.swap_out(flat, flat.numel(), _DTYPES[t.dtype], codec, hidden_f, hidden_b)
        # a raw (NONE) offload reads t on the library's copy stream: t's memory must not be
        # reused before that copy ends -> order a torch stream after it and tie t to it.  A
        # compressed swap-out reads t only on the current stream (the codec kernels), so torch's
        # stream-ordered allocator already keeps t alive long enough, and nothing here waits.
        if h.codec() == C.NONE:
            h.record_out(self.keep)
            t.record_stream(self.keep)
        return h

    def swap_in(self, h, out: torch.Tensor, stream: torch.cuda.Stream):
        h.swap_in(out.view(-1), stream=stream)

    @staticmethod
    def codec(h) -> int:
        return h.codec()  # known when swap_out returns: no wait

    @staticmethod
    def info(h) -> tuple[int, int]:
        q = h.query()  # waits until the swap-out's copies are issued
        return q["codec"], q["bytes"]

    @staticmethod
    def free(h):
        h.close()


@dataclasses.dataclass
class _Rec:
    index: int
    shape: torch.Size
    dtype: torch.dtype
    device: torch.device
    nbytes: int
    handle: object = None
    refs: int = 1
    restored: torch.Tensor | None = None
    ready: torch.cuda.Event | None = None
    codec: int = -1
    comp_bytes: int = 0
    original: torch.Tensor | None = None
    ref: object = None  # weak reference to the saved tensor object (identity for deduplication)


class _Prof:
    __slots__ = ("t", "index")

    def __init__(self, t, index):
        self.t, self.index = t, index


class SwapSaver:
    """Context manager installing saved-tensor hooks that swap activations through libcswap.

        saver = SwapSaver("auto")
        saver.profile(lambda: step(model, x))   # optional: measure Hidden_f / Hidden_b
        with saver:
            loss = model(x).sum()
        loss.backward()                         # restores (and prefetches) on use
    """

    def __init__(self, policy="auto", min_bytes: int = 1 << 20, prefetch: bool = True, backend=None,
                 verify: bool = False, reprofile_every: int = 0):
        if not (isinstance(policy, int) or policy in ("resident", *POLICIES)):
            raise ValueError(f"unknown policy {policy!r}")
        self.policy = policy
        self.min_bytes = min_bytes
        self.prefetch = prefetch
        self.backend = backend
        self.verify = verify  # debug: keep a device copy of every swapped tensor, compare on use
        self.mismatches: list[tuple[int, int]] = []
        self.hidden: list[tuple[float, float]] | None = None
        # online re-profiling (NEXT-2; PAPER.md:118 "sparsity ... per epoch", :156-162): with
        # reprofile_every = N > 0 the AUTO policy probes and decides only on every N-th step
        # (a profiling step) and replays the stored execution plan — one codec per tensor index —
        # on the others, which then skip the probe and its host synchronisation
        self.reprofile_every = reprofile_every
        self.step_index = -1
        self.plan: list[int] | None = None
        self.plan_history: list[tuple[int, list[int]]] = []
        self._order: list[_Rec] = []
        self._live: dict = {}
        self._ctx = None
        self._prof = None
        self.stats = {}

    # ---- candidates -----------------------------------------------------------------------
    def _candidate(self, t: torch.Tensor) -> bool:
        if not isinstance(t, torch.Tensor) or t.dtype not in _DTYPES or not t.is_contiguous():
            return False
        if t.requires_grad and t.is_leaf:  # parameters (and inputs that want grads) stay resident
            return False
        if t.numel() * t.element_size() < self.min_bytes:
            return False
        return self.backend.accepts(t) if self.backend is not None else t.is_cuda

    @staticmethod
    def _key(t: torch.Tensor):
        return (t.untyped_storage().data_ptr(), t.storage_offset(), t.numel(), t.dtype, t._version)

    # ---- hooks ------------------------------------------------------------------------------
    def __enter__(self):
        if self.policy != "resident" and self.backend is None:
            self.backend = CSwapBackend()
        self._order, self._live = [], {}
        self.stats = {"swapped": 0, "raw_bytes": 0, "comp_bytes": 0, "codecs": []}
        self.step_index += 1
        self._profiling = (self.policy == "auto" and (self.reprofile_every <= 0 or self.plan is None
                                                      or self.step_index % self.reprofile_every == 0))
        self._ctx = torch.autograd.graph.saved_tensors_hooks(self._pack, self._unpack)
        self._ctx.__enter__()
        return self

    def __exit__(self, *exc):
        self._ctx.__exit__(*exc)
        self._ctx = None
        if self.policy == "auto" and self.reprofile_every > 0 and self._profiling:
            self.plan = list(self.stats["codecs"])
            self.plan_history.append((self.step_index, self.plan))
        return False

    def _pack(self, t):
        if self._prof is not None:
            return self._prof_pack(t)
        if self.policy == "resident" or not self._candidate(t):
            return t
        key = self._key(t)
        rec = self._live.get(key)
        # the same activation saved by a second op (ReLU output -> conv input) is the same live
        # tensor object; a key match with a dead object is a NEW tensor the allocator placed where
        # a swapped-out (and freed) one of the same size used to be
        if rec is not None and rec.ref is not None and rec.ref() is t:
            rec.refs += 1
            return rec
        i = len(self._order)
        hf, hb = self.hidden[i] if self.hidden and i < len(self.hidden) else (0.0, 0.0)
        codec = self.policy if isinstance(self.policy, int) else POLICIES[self.policy]
        if codec == C.AUTO and not self._profiling and self.plan is not None and i < len(self.plan):
            codec = self.plan[i]
        rec = _Rec(i, t.shape, t.dtype, t.device, t.numel() * t.element_size())
        rec.ref = weakref.ref(t)
        if self.verify:
            rec.original = t.detach().clone()
        rec.handle = self.backend.swap_out(t, codec, hf, hb)
        # the codec is known at once; the container size only once the swap-out has run, so it is
        # read when the record is released (reading it here would make every save wait for its
        # compression, and the forward pass could no longer run ahead of the GPU)
        rec.codec = self.backend.codec(rec.handle) if hasattr(self.backend, "codec") else \
            self.backend.info(rec.handle)[0]
        self._live[key] = rec
        self._order.append(rec)
        self.stats["swapped"] += 1
        self.stats["raw_bytes"] += rec.nbytes
        self.stats["codecs"].append(rec.codec)
        return rec

    def _restore(self, rec: _Rec, stream):
        out = torch.empty(rec.shape, dtype=rec.dtype, device=rec.device)
        cur = torch.cuda.current_stream(rec.device) if rec.device.type == "cuda" else None
        if stream is not None and cur is not None and stream != cur:
            stream.wait_stream(cur)  # `out` was allocated in the current stream's order
            out.record_stream(stream)
        self.backend.swap_in(rec.handle, out, stream if stream is not None else cur)
        if stream is not None and cur is not None:
            rec.ready = torch.cuda.Event()
            rec.ready.record(stream)
        rec.restored = out

    def _unpack(self, rec):
        if isinstance(rec, _Prof):
            return self._prof_unpack(rec)
        if not isinstance(rec, _Rec):
            return rec
        if rec.restored is None:
            self._restore(rec, None)
        elif rec.ready is not None:
            torch.cuda.current_stream(rec.device).wait_event(rec.ready)
        t = rec.restored
        if rec.original is not None:
            if not torch.equal(t.view(torch.int16 if t.element_size() == 2 else torch.int32),
                               rec.original.view(torch.int16 if t.element_size() == 2 else torch.int32)):
                self.mismatches.append((rec.index, rec.codec))
        rec.refs -= 1
        if rec.refs == 0:  # every saving op has its copy: drop ours and the host container
            rec.comp_bytes = self.backend.info(rec.handle)[1]
            self.stats["comp_bytes"] += rec.comp_bytes
            rec.restored = None
            rec.original = None
            self.backend.free(rec.handle)
            rec.handle = None
            self._live = {k: v for k, v in self._live.items() if v is not rec}
        if self.prefetch:
            nxt = next((r for r in reversed(self._order[:rec.index]) if r.handle is not None and r.restored is None),
                       None)
            if nxt is not None:
                self._restore(nxt, getattr(self.backend, "prefetch", None))
        return t

    # ---- tensor profiler (Hidden_f / Hidden_b) ---------------------------------------------
    def _prof_pack(self, t):
        if not self._candidate(t):
            return t
        key = self._key(t)
        if key in self._prof["keys"]:
            return _Prof(t, self._prof["keys"][key])
        i = len(self._prof["fwd"])
        self._prof["keys"][key] = i
        e = torch.cuda.Event(enable_timing=True)
        e.record()
        self._prof["fwd"].append(e)
        return _Prof(t, i)

    def _prof_unpack(self, p: _Prof):
        bwd = self._prof["bwd"]
        if p.index not in bwd:
            e = torch.cuda.Event(enable_timing=True)
            e.record()
            bwd[p.index] = e
        return p.t

    def profile(self, step_fn) -> list[tuple[float, float]]:
        """One step with events at every candidate's save and first use; sets and returns
        self.hidden = [(Hidden_f, Hidden_b)] in seconds, indexed in save order.  `step_fn` must
        run forward AND backward inside itself; the hooks are installed around the whole call."""
        if self.backend is None and self.policy != "resident":
            self.backend = CSwapBackend()
        self._prof = {"keys": {}, "fwd": [], "bwd": {}}
        end_f = torch.cuda.Event(enable_timing=True)
        ctx = torch.autograd.graph.saved_tensors_hooks(self._pack, self._unpack)
        try:
            with ctx:
                step_fn(lambda: end_f.record())
        finally:
            prof, self._prof = self._prof, None
        torch.cuda.synchronize()
        fwd, bwd, m = prof["fwd"], prof["bwd"], len(prof["fwd"])
        hidden = []
        for i in range(m):
            hf = fwd[i].elapsed_time(fwd[i + 1] if i + 1 < m else end_f) * 1e-3
            hb = bwd[i + 1].elapsed_time(bwd[i]) * 1e-3 if (i in bwd and i + 1 in bwd) else 0.0
            hidden.append((max(hf, 0.0), max(hb, 0.0)))
        self.hidden = hidden
        return hidden
