"""Stage / pipeline bindings over libsq (marshalling only) + device-resident model builder.

``Layer`` owns the four quantized linears of one decoder layer (P:160 linear
set; R11).  ``build_layers`` creates synthetic OPT/BLOOM-shaped
layers directly in HBM with the seeded counter generator (synth/), quantizing
and packing them with the library's own kernels (load-time path).
"""
from __future__ import annotations

import ctypes

import torch

from . import (P, QLinear, SQ_DECODE, SQ_PREFILL, _L, _check, _ptr, _stream, sq_attn, sq_layer, sq_plan,
               sq_run_stats)


class Layer:
    def __init__(self, bits: int, act: int, qkv: QLinear, o: QLinear, fc1: QLinear, fc2: QLinear):
        self.bits, self.act = bits, act
        self.qkv, self.o, self.fc1, self.fc2 = qkv, o, fc1, fc2

    def c_struct(self) -> sq_layer:
        return sq_layer(self.bits, self.act, self.qkv.c, self.o.c, self.fc1.c, self.fc2.c)

    def nbytes(self) -> int:
        return sum(l.nbytes() for l in (self.qkv, self.o, self.fc1, self.fc2))


def layer_array(layers: list[Layer]):
    return (sq_layer * len(layers))(*[l.c_struct() for l in layers])


def build_layers(n_layers: int, h1: int, h2: int, bits: list[int], act: int = 0, bias: bool = True,
                 layer_offset: int = 0, device: str = "cuda", stream=None) -> list[Layer]:
    """Synthetic layers (W ~ N(0, 1/K) + 0.1 % outliers) built in HBM."""
    import synth
    layers = []
    dims = {"qkv": (3 * h1, h1), "o": (h1, h1), "fc1": (h2, h1), "fc2": (h1, h2)}
    scratch = torch.empty(max(n * k for n, k in dims.values()), dtype=torch.float16, device=device)
    s = torch.cuda.current_stream() if stream is None else stream
    for i in range(n_layers):
        l = layer_offset + i
        b = int(bits[i])
        lins = {}
        for name, (n, k) in dims.items():
            seed = synth.weight_seed(l, name)
            if b == 16:
                w = torch.empty((n, k), dtype=torch.float16, device=device)
                synth.device_weight_f16(w.data_ptr(), seed, n, k, s.cuda_stream)
            else:
                w = scratch[: n * k].view(n, k)
                synth.device_weight_f16(w.data_ptr(), seed, n, k, s.cuda_stream)
            bvec = None
            if bias:
                bvec = torch.from_numpy(synth.bias_f16(seed, n)).to(device)
            lins[name] = QLinear.from_fp16(w, b, bvec, stream=s)
        layers.append(Layer(b, act, lins["qkv"], lins["o"], lins["fc1"], lins["fc2"]))
    torch.cuda.synchronize()
    return layers


# ---------------------------------------------------------------- a5
def sq_stage_workspace_bytes(layers: list[Layer], max_tokens: int) -> int:
    arr = layer_array(layers)
    return int(_L.sq_stage_workspace_bytes(arr, len(layers), max_tokens))


class StageWorkspace:
    def __init__(self, layers: list[Layer], max_tokens: int, device="cuda"):
        self.buf = torch.zeros(sq_stage_workspace_bytes(layers, max_tokens) + 256, dtype=torch.uint8, device=device)
        off = (-self.buf.data_ptr()) % 256
        self.ptr = self.buf.data_ptr() + off
        self.nbytes = self.buf.numel() - off


def sq_stage_forward(layers: list[Layer], phase: int, x_in: torch.Tensor, x_out: torch.Tensor,
                     ws: StageWorkspace, qkv_dbg: torch.Tensor | None = None, stream=None, arr=None) -> torch.Tensor:
    """a5: run this stage's layers on x fp32 [tokens, h1] (x_in and x_out may alias)."""
    arr = layer_array(layers) if arr is None else arr
    _check(_L.sq_stage_forward(arr, len(layers), phase, _ptr(x_in), x_in.shape[0], _ptr(x_out), _ptr(qkv_dbg),
                               ctypes.c_void_p(ws.ptr), ws.nbytes, _stream(stream)))
    return x_out


class KVCache:
    """Device KV cache of a stage (f3): per layer K, V fp16 [n_seq, max_len, h1] (P:162 sizing)."""

    def __init__(self, n_layers: int, n_seq: int, max_len: int, h1: int, device="cuda"):
        self.k = torch.zeros((n_layers, n_seq, max_len, h1), dtype=torch.float16, device=device)
        self.v = torch.zeros_like(self.k)
        self.n_seq, self.max_len, self.h1 = n_seq, max_len, h1
        self._kp = (P * n_layers)(*[self.k[l].data_ptr() for l in range(n_layers)])
        self._vp = (P * n_layers)(*[self.v[l].data_ptr() for l in range(n_layers)])

    def ctx(self, n_heads: int, seq0: int, nseq: int, seq_len: int, pos0: int) -> sq_attn:
        return sq_attn(n_heads, self.max_len, self.n_seq, self._kp, self._vp, seq0, nseq, seq_len, pos0)


def sq_stage_forward_attn(layers: list[Layer], phase: int, x_in: torch.Tensor, x_out: torch.Tensor,
                          ws: StageWorkspace, cache: KVCache, n_heads: int, seq0: int, nseq: int, seq_len: int,
                          pos0: int, stream=None, arr=None) -> torch.Tensor:
    """a5 with real attention (f3): rows of x are (sequence, position), tokens = nseq * seq_len."""
    arr = layer_array(layers) if arr is None else arr
    ctx = cache.ctx(n_heads, seq0, nseq, seq_len, pos0)
    _check(_L.sq_stage_forward_attn(arr, len(layers), phase, ctypes.byref(ctx), _ptr(x_in), x_in.shape[0],
                                    _ptr(x_out), ctypes.c_void_p(ws.ptr), ws.nbytes, _stream(stream)))
    return x_out


def sq_layernorm_f32(x: torch.Tensor, y: torch.Tensor, stream=None) -> torch.Tensor:
    _check(_L.sq_layernorm_f32(_ptr(x), x.shape[0], x.shape[1], _ptr(y), _stream(stream)))
    return y


# ---------------------------------------------------------------- a6
class Plan:
    """Host-side plan (per-layer bits, layer->stage partition, micro-batch sizes)."""

    def __init__(self, bits: list[int], stage_of_layer: list[int], hidden: int, ffn: int, B: int, eta: int,
                 xi: int, prompt_len: int, n_decode: int, group: int = 128, n_heads: int = 0, kappa: int = 1,
                 tp: int = 1):
        self.bits = [int(b) for b in bits]
        self.stage_of_layer = [int(s) for s in stage_of_layer]
        self.n_layers = len(bits)
        self.n_stages = max(self.stage_of_layer) + 1
        self.hidden, self.ffn, self.B, self.eta, self.xi = hidden, ffn, B, eta, xi
        self.prompt_len, self.n_decode, self.group = prompt_len, n_decode, group
        self._bits = (ctypes.c_int32 * self.n_layers)(*self.bits)
        self._sol = (ctypes.c_int32 * self.n_layers)(*self.stage_of_layer)
        self.n_heads, self.kappa, self.tp = n_heads, kappa, max(1, tp)
        self.c = sq_plan(self.n_layers, self.n_stages, hidden, ffn, group, self._bits, self._sol, B, eta, xi,
                         prompt_len, n_decode, n_heads, kappa, tp)

    @property
    def n_ranks(self) -> int:
        return self.n_stages * self.tp

    def layers_of(self, rank: int) -> list[int]:
        """layer indices held by global rank `rank` (stage rank // tp)"""
        return [l for l, s in enumerate(self.stage_of_layer) if s == rank // self.tp]


def sq_plan_check(plan: Plan) -> None:
    _check(_L.sq_plan_check(ctypes.byref(plan.c)))


def sq_pipeline_schedule(plan: Plan, rank: int) -> list[dict]:
    """Host-only: the op sequence `rank` executes in sq_pipeline_run (see sq.h)."""
    from . import SQ_OP_NAMES, sq_sched_op
    n = int(_L.sq_pipeline_schedule(ctypes.byref(plan.c), rank, None, 0))
    if n < 0:
        raise ValueError("invalid plan")
    arr = (sq_sched_op * max(n, 1))()
    _L.sq_pipeline_schedule(ctypes.byref(plan.c), rank, arr, n)
    return [{"kind": SQ_OP_NAMES[o.kind], "item": o.item, "phase": o.phase, "t": o.t, "slot": o.slot,
             "peer": o.peer, "seq0": o.seq0, "nseq": o.nseq, "rows": o.rows} for o in arr[:n]]


class Comm:
    def __init__(self, handle: int):
        self.h = ctypes.c_void_p(handle)

    @classmethod
    def local(cls, nstages: int) -> "Comm":
        h = ctypes.c_void_p()
        _check(_L.sq_comm_init_local(ctypes.byref(h), nstages))
        return cls(h.value)

    @classmethod
    def mesh(cls, uid: bytes, n_stages: int, tp: int, rank: int) -> "Comm":
        """P x tp mesh (f4): stage rings + one TP communicator per stage (sq_comm_init_mesh)."""
        h = ctypes.c_void_p()
        buf = (ctypes.c_uint8 * len(uid)).from_buffer_copy(uid)
        _check(_L.sq_comm_init_mesh(ctypes.byref(h), buf, n_stages, tp, rank))
        return cls(h.value)

    @classmethod
    def nccl(cls, uid: bytes, nranks: int, rank: int) -> "Comm":
        h = ctypes.c_void_p()
        buf = (ctypes.c_uint8 * len(uid)).from_buffer_copy(uid)
        _check(_L.sq_comm_init(ctypes.byref(h), buf, nranks, rank))
        return cls(h.value)

    def destroy(self) -> None:
        if self.h:
            _L.sq_comm_destroy(self.h)
            self.h = ctypes.c_void_p()


def sq_comm_get_unique_id() -> bytes:
    n = int(_L.sq_comm_unique_id_bytes())
    buf = (ctypes.c_uint8 * n)()
    _check(_L.sq_comm_get_unique_id(buf))
    return bytes(buf)


def _flat(layers):
    """list[Layer] -> itself; TP shard sets list[list[Layer]] ([tp][n_layers]) -> flattened, set-major"""
    if layers and isinstance(layers[0], (list, tuple)):
        return [l for s in layers for l in s], len(layers[0])
    return layers, len(layers)


class PipelineWorkspace:
    def __init__(self, plan: Plan, layers, rank: int, device="cuda"):
        arr = layer_array(_flat(layers)[0])
        n = int(_L.sq_pipeline_workspace_bytes(ctypes.byref(plan.c), arr, rank))
        if n == 0:
            raise ValueError("invalid plan/layers for workspace query")
        self.buf = torch.zeros(n + 256, dtype=torch.uint8, device=device)
        off = (-self.buf.data_ptr()) % 256
        self.ptr = self.buf.data_ptr() + off
        self.nbytes = n


def sq_pipeline_run(plan: Plan, rank: int, layers, comm: Comm | None, x0: torch.Tensor | None,
                    out: torch.Tensor | None, ws: PipelineWorkspace, stream=None, arr=None) -> dict:
    """a6: run the whole generation (prefill + n_decode steps) for this rank (rank -1: all stages).
    TP plans (plan.tp > 1): layers = this rank's shards, or for rank -1 the [tp][n_layers] shard sets."""
    flat, n_layers = _flat(layers)
    arr = layer_array(flat) if arr is None else arr
    st = sq_run_stats()
    _check(_L.sq_pipeline_run(ctypes.byref(plan.c), rank, arr, n_layers, comm.h if comm else None, _ptr(x0),
                              _ptr(out), ctypes.c_void_p(ws.ptr), ws.nbytes, ctypes.byref(st), _stream(stream)))
    return {"t_total_ms": st.t_total_ms, "t_prefill_ms": st.t_prefill_ms, "t_decode_ms": st.t_decode_ms,
            "tokens_per_s": st.tokens_per_s, "bytes_sent": st.bytes_sent, "gpu_launches": st.gpu_launches,
            "host_enqueue_ms": st.host_enqueue_ms, "graph_replays": st.graph_replays}


# ---------------------------------------------------------------- f4: tensor-parallel stage (R27)
def tp_shard_fp16(name: str, w: torch.Tensor, bias: torch.Tensor | None, r: int, T: int):
    """Shard r of T of one linear (sq.h f4 split): qkv / fc1 by output rows (qkv: the same row slice of
    each of q, k, v), o / fc2 by input columns with the bias on rank 0 only.  -> (w fp16, bias)."""
    n, k = w.shape
    if name == "qkv":
        h = n // 3
        s = h // T
        idx = [slice(j * h + r * s, j * h + (r + 1) * s) for j in range(3)]
        ws = torch.cat([w[i] for i in idx])
        b = None if bias is None else torch.cat([bias[i] for i in idx])
    elif name == "fc1":
        s = n // T
        ws, b = w[r * s:(r + 1) * s], None if bias is None else bias[r * s:(r + 1) * s]
    else:
        s = k // T
        ws, b = w[:, r * s:(r + 1) * s], (bias if r == 0 else None)
    return ws.contiguous(), None if b is None else b.contiguous()


def build_tp_layers(n_layers: int, h1: int, h2: int, bits: list[int], T: int, act: int = 0, bias: bool = True,
                    layer_offset: int = 0, device: str = "cuda", ranks=None) -> list[list[Layer]]:
    """The synthetic layers of build_layers split into T tensor-parallel shards: [rank][layer] for the
    ranks in `ranks` (default all; a real TP rank builds only its own)."""
    import synth
    ranks = list(range(T)) if ranks is None else list(ranks)
    dims = {"qkv": (3 * h1, h1), "o": (h1, h1), "fc1": (h2, h1), "fc2": (h1, h2)}
    s = torch.cuda.current_stream()
    out = [[] for _ in ranks]
    for i in range(n_layers):
        l = layer_offset + i
        b = int(bits[i])
        lins = [{} for _ in ranks]
        for name, (n, k) in dims.items():
            seed = synth.weight_seed(l, name)
            w = torch.empty((n, k), dtype=torch.float16, device=device)
            synth.device_weight_f16(w.data_ptr(), seed, n, k, s.cuda_stream)
            bvec = torch.from_numpy(synth.bias_f16(seed, n)).to(device) if bias else None
            for j, r in enumerate(ranks):
                ws, bs = tp_shard_fp16(name, w, bvec, r, T)
                lins[j][name] = QLinear.from_fp16(ws, b, bs, stream=s)
        for j in range(len(ranks)):
            out[j].append(Layer(b, act, lins[j]["qkv"], lins[j]["o"], lins[j]["fc1"], lins[j]["fc2"]))
    torch.cuda.synchronize()
    return out


class TpWorkspace:
    def __init__(self, shard_sets: list[list[Layer]], max_tokens: int, device="cuda"):
        arr = layer_array([l for s in shard_sets for l in s])
        n = int(_L.sq_stage_tp_workspace_bytes(arr, sum(len(s) for s in shard_sets), max_tokens))
        if n == 0:
            raise ValueError("invalid shards for workspace query")
        self.buf = torch.zeros(n + 256, dtype=torch.uint8, device=device)
        off = (-self.buf.data_ptr()) % 256
        self.ptr = self.buf.data_ptr() + off
        self.nbytes = n


def sq_stage_forward_tp(shard_sets: list[list[Layer]], phase: int, x_in: torch.Tensor, x_out: torch.Tensor,
                        ws: TpWorkspace, T: int, tp_rank: int = -1, comm: Comm | None = None,
                        caches: list[KVCache] | None = None, n_heads: int = 0, seq0: int = 0, nseq: int = 0,
                        seq_len: int = 0, pos0: int = 0, stream=None) -> torch.Tensor:
    """f4: one stage under T-way TP.  tp_rank -1: virtual TP (shard_sets = all T ranks' layers on this
    device); tp_rank >= 0: this rank's single shard set, partial sums all-reduced over `comm`.  With
    `caches` (one KVCache of width h1/T per shard set) the layers run causal attention over n_heads
    heads (n_heads / T per rank)."""
    n_layers = len(shard_sets[0])
    arr = layer_array([l for s in shard_sets for l in s])
    ctx = None
    if caches is not None:
        ctx = (sq_attn * len(caches))(*[c.ctx(n_heads // T, seq0, nseq, seq_len, pos0) for c in caches])
    _check(_L.sq_stage_forward_tp(arr, n_layers, T, tp_rank, comm.h if comm else None, phase, ctx, _ptr(x_in),
                                  x_in.shape[0], _ptr(x_out), ctypes.c_void_p(ws.ptr), ws.nbytes, _stream(stream)))
    return x_out
