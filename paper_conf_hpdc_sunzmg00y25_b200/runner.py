"""Synthetic decoder-only LLM runner with FT2 protection on its critical layers.

This is the *host model* around FT2's hot path (attention,
norms, activations, embeddings and sampling run as plain torch ops -- they
are not part of the method).  The method itself runs in libft2.so:

* critical layers (Table 1): OPT/GPT-J
  v_proj, out_proj, fc2; Llama/Qwen2 v_proj, o_proj, up_proj, down_proj;
* prefill (first token): each critical layer's output is reduced to per-
  sequence bounds x2 and its non-finite values are corrected
  (ft2_bounds_from_prefill);
* every decode step: each critical layer's output is checked and clipped
  (PAPER.md L259-L272), either
    - "standalone": cuBLAS linear + ft2_protect (the paper's own structure:
      a fused clamp/nan_to_num op called after the layer, L272), or
    - "fused": ft2_protect_fused_gemm with the check in the tcgen05 GEMM
      epilogue (no extra kernel, no extra HBM pass);
* "off" is the unprotected baseline (cuBLAS linears, no FT2 work), and
  "fused_plain" runs the same tcgen05 GEMM without the check (isolates the
  epilogue's cost).

Weights are seeded synthetic (ft2_synth recipe, scaled 2^-ceil(log2 sqrt K));
no checkpoint is loaded.  The first-token pass and the decode step are each
captured once per mode into a CUDA graph (static prompt / token buffers) and
replayed: one prefill replay and G-1 decode replays per request.
"""
from __future__ import annotations

import dataclasses

import torch
import torch.nn.functional as F

import ft2_synth

from . import ft2 as F2
from ._lib import FT2_GEMM_CHECK, FT2_GEMM_PLAIN, FT2_GEMM_W_STATIC

MODES = ("off", "standalone", "fused", "fused_plain")
FUSED_MAX_M = 128


@dataclasses.dataclass(frozen=True)
class ModelConfig:
    arch: str              # "opt" | "llama"
    hidden: int
    ffn: int
    n_layers: int
    n_heads: int
    vocab: int
    max_pos: int = 2048
    bias: bool = True

    @property
    def head_dim(self):
        return self.hidden // self.n_heads

    def linears(self):
        """Block linear layers in order: (name, out_features, in_features, critical)."""
        h, f = self.hidden, self.ffn
        if self.arch == "opt":
            return [("q_proj", h, h, False), ("k_proj", h, h, False), ("v_proj", h, h, True),
                    ("out_proj", h, h, True), ("fc1", f, h, False), ("fc2", h, f, True)]
        return [("q_proj", h, h, False), ("k_proj", h, h, False), ("v_proj", h, h, True),
                ("o_proj", h, h, True), ("gate_proj", f, h, False), ("up_proj", f, h, True),
                ("down_proj", h, f, True)]

    def critical_names(self):
        return [n for n, _, _, c in self.linears() if c]

    def coverage_names(self, coverage: str = "ft2"):
        """Linear layers a protection scheme covers (Table 1).

        "ft2": the critical layers (the heuristic of Sec. 4.1.2); "maximals":
        OUT_PROJ/FC2/DOWN_PROJ; "globalclipper": V_PROJ/OUT_PROJ; "all": every
        linear layer; "none": Ranger's coverage of linear layers (it protects
        activation layers only, L315).  Llama's o_proj plays OUT_PROJ's role.
        """
        role = {"o_proj": "out_proj"}
        sets = {"ft2": None, "all": None, "none": set(),
                "maximals": {"out_proj", "fc2", "down_proj"}, "globalclipper": {"v_proj", "out_proj"}}
        if coverage not in sets:
            raise ValueError(f"unknown coverage {coverage!r}; one of {sorted(sets)}")
        if coverage == "ft2":
            return self.critical_names()
        if coverage == "all":
            return [n for n, _, _, _ in self.linears()]
        return [n for n, _, _, _ in self.linears() if role.get(n, n) in sets[coverage]]

    def critical_widths(self):
        """Output width of every protected layer, block-major (the bounds/site layer ids)."""
        per = [o for _, o, _, c in self.linears() if c]
        return per * self.n_layers

    def linear_widths(self):
        per = [o for _, o, _, _ in self.linears()]
        return per * self.n_layers


# Shapes (SURVEY.md §0 external facts: HF config defaults / public model cards).
CONFIGS = {
    "opt-125m": ModelConfig("opt", 768, 3072, 12, 12, 50272),
    "opt-1.3b": ModelConfig("opt", 2048, 8192, 24, 32, 50272),
    "opt-2.7b": ModelConfig("opt", 2560, 10240, 32, 32, 50272),
    "opt-6.7b": ModelConfig("opt", 4096, 16384, 32, 32, 50272),
    "llama-2-7b": ModelConfig("llama", 4096, 11008, 32, 32, 32000, 4096, False),
    "llama-2-13b": ModelConfig("llama", 5120, 13824, 40, 40, 32000, 4096, False),
}


def _w(shape, tau, seed, device, K=None, outliers=True, dtype=torch.bfloat16):
    sl = ft2_synth.weight_scale_log2(K) if K else 0
    t = ft2_synth.gen_bf16_torch(shape, tau, seed, scale_log2=sl, device=device, outliers=outliers)
    return t if dtype == torch.bfloat16 else t.to(dtype)   # FP16 model: the same values, rounded


class Block:
    def __init__(self, cfg: ModelConfig, idx: int, seed: int, device, outliers: bool = True,
                 dtype=torch.bfloat16):
        self.cfg = cfg
        self.idx = idx
        tau0 = 1000 + 64 * idx
        self.w = {}
        self.b = {}
        for j, (name, o, i, _) in enumerate(cfg.linears()):
            self.w[name] = _w((o, i), tau0 + 2 * j, seed, device, K=i, outliers=outliers, dtype=dtype)
            self.b[name] = _w((o,), tau0 + 2 * j + 1, seed, device, outliers=outliers, dtype=dtype) if cfg.bias else None
        # horizontally fused projections (same weights; the per-layer tensors
        # become views into the fused ones): qkv, and Llama's gate_up
        self.groups = {"qkv": ["q_proj", "k_proj", "v_proj"]}
        if cfg.arch == "llama":
            self.groups["gate_up"] = ["gate_proj", "up_proj"]
        self.wf, self.bf = {}, {}
        for g, names in self.groups.items():
            self.wf[g] = torch.cat([self.w[n] for n in names])
            self.bf[g] = torch.cat([self.b[n] for n in names]) if cfg.bias else None
            r0 = 0
            for n in names:
                o = self.w[n].shape[0]
                self.w[n] = self.wf[g][r0:r0 + o]
                if cfg.bias:
                    self.b[n] = self.bf[g][r0:r0 + o]
                r0 += o
        h = cfg.hidden
        self.ln1_w = torch.ones(h, dtype=dtype, device=device)
        self.ln2_w = torch.ones(h, dtype=dtype, device=device)
        self.ln1_b = torch.zeros(h, dtype=dtype, device=device) if cfg.arch == "opt" else None
        self.ln2_b = torch.zeros(h, dtype=dtype, device=device) if cfg.arch == "opt" else None


class FT2State:
    """Per-request FT2 state: bounds [L_crit, B, 2], counters, workspace."""

    def __init__(self, n_crit: int, B: int, device, dtype=torch.bfloat16):
        self.bounds = torch.zeros((n_crit, B, 2), dtype=dtype, device=device)
        self.keys = torch.zeros((n_crit, B, 2), dtype=torch.int32, device=device)
        self.corrected = torch.zeros((n_crit, B), dtype=torch.int32, device=device)
        self.nonfinite = torch.zeros((n_crit, B), dtype=torch.int32, device=device)
        self.ws = F2.make_workspace(B, device=device)

    def reset_counters(self):
        self.corrected.zero_()
        self.nonfinite.zero_()


class Runner:
    """Batched greedy generation with FT2 on the critical layers."""

    def __init__(self, cfg: ModelConfig, batch: int, prompt_len: int, gen_len: int, seed: int = 1,
                 device="cuda", scale: float = 2.0, coverage: str = "ft2", fuse_proj: bool | None = None,
                 share: "Runner | None" = None, outliers: bool = True, dtype=torch.bfloat16):
        """share: another Runner of the same config, batch and lengths whose
        weights, KV caches and static token / site buffers this one reuses
        (no copy; see with_coverage).  Runners sharing buffers must not run
        concurrently.  outliers=False builds the weights and embeddings without
        the synthetic recipe's planted 2**-10 outliers: the
        fault-injection campaign's model, whose fault-free activation range is
        stable from the first token on (the premise of first-token bounds,
        PAPER.md L223-L233), unlike the heavy-tailed outlier model.  dtype:
        torch.bfloat16 (BASELINE) or torch.float16 (the paper's precision,
        PAPER.md L282) for the whole model, FT2's kernels and bounds included."""
        assert dtype in (torch.bfloat16, torch.float16), dtype
        self.dt = dtype
        self.cfg = cfg
        self.B = batch
        self.T = prompt_len
        self.G = gen_len
        self.Tmax = prompt_len + gen_len
        self.scale = scale
        self.device = torch.device(device)
        dv = self.device
        h = cfg.hidden
        if share is not None:
            assert (share.cfg, share.B, share.T, share.G, share.dt) == (cfg, batch, prompt_len, gen_len, dtype)
            for a in ("embed", "pos_embed", "blocks", "lnf_w", "lnf_b", "lm_head"):
                setattr(self, a, getattr(share, a))
        else:
            self.embed = _w((cfg.vocab, h), 1, seed, dv, outliers=outliers, dtype=dtype)
            self.pos_embed = _w((cfg.max_pos + 2, h), 2, seed, dv, outliers=outliers, dtype=dtype) \
                if cfg.arch == "opt" else None
            self.blocks = [Block(cfg, i, seed, dv, outliers=outliers, dtype=dtype) for i in range(cfg.n_layers)]
            self.lnf_w = torch.ones(h, dtype=dtype, device=dv)
            self.lnf_b = torch.zeros(h, dtype=dtype, device=dv) if cfg.arch == "opt" else None
            self.lm_head = self.embed if cfg.arch == "opt" else _w((cfg.vocab, h), 3, seed, dv, K=h,
                                                                   outliers=outliers, dtype=dtype)
        self.coverage = coverage
        # fuse_proj: fused q/k/v (and Llama gate/up) projections, one GEMM per
        # group; the protected layer of a group (v_proj, up_proj) is a column
        # slice whose check runs in the fused GEMM's epilogue (col_begin/
        # col_end).  Off by default: at the fused OPT-1.3B QKV shape (N = 6144,
        # K = 2048, M = 32) the tcgen05 decode GEMM runs 15.4-20.2 us in situ
        # against cuBLAS's 13.5 us (profiles/r1_qkv_splitk.txt), so fusing
        # helps the unprotected baseline more than FT2 (measured 8.4 % FT2
        # overhead fused vs 2.8 % unfused).  Fault campaigns address sites per
        # linear layer and need fuse_proj=False.
        import os
        if fuse_proj is None:   # FT2_FUSE_PROJ=1 flips the default (experiments)
            fuse_proj = os.environ.get("FT2_FUSE_PROJ", "0") == "1"
        self.fuse_proj = fuse_proj
        # critical layers whose decode check runs as cuBLAS + ft2_protect even
        # in "fused" mode (FT2_STANDALONE_LAYERS="v_proj,out_proj", experiments)
        self.standalone_layers = set(filter(None, os.environ.get("FT2_STANDALONE_LAYERS", "").split(",")))
        # decoder norms and MLP activations through libft2's host-model
        # kernels (they trigger PDL dependents on entry, so the v_proj / fc2 /
        # down_proj GEMM prologue overlaps them); FT2_HOST_NORM=0 keeps
        # torch's kernels (experiments)
        self.host_norm = os.environ.get("FT2_HOST_NORM", "1") == "1"
        self.host_act = self.host_norm and os.environ.get("FT2_HOST_ACT", "1") == "1"
        # L2 prefetch hint of the decode GEMMs (ft2_protect_fused_gemm_ex): a
        # fused critical-layer GEMM pulls the weights of the next one into L2
        # once its own operands have landed.  Default (FT2_L2_PREFETCH=2): only
        # v_proj, for out_proj / o_proj -- the layer after attention, which is
        # latency-bound and triggers no PDL, so out_proj otherwise pays its whole
        # weight fetch after it (session e, OPT-1.3B in situ, two A/B pairs:
        # 16 970 -> 16 990 protected tok/s, decode step 1.744 -> 1.741 ms).
        # FT2_L2_PREFETCH=1 hints every layer (slower: the prefetch of fc2's
        # 34 MB competes with fc1's own stream; 16 928 tok/s), 0 none.
        mode = os.environ.get("FT2_L2_PREFETCH", "2")
        self.l2_prefetch = mode in ("1", "2")
        self.l2_prefetch_after_attn = mode == "2"
        self.crit_names = cfg.coverage_names(coverage)   # protected layers of one block
        self.lin_names = [n for n, _, _, _ in cfg.linears()]
        self.n_crit = len(self.crit_names) * cfg.n_layers
        self.state = FT2State(self.n_crit, batch, dv, dtype)
        H, D = cfg.n_heads, cfg.head_dim
        # buffers a with_coverage() clone shares with its parent (graphs bake in
        # their addresses; runs are sequential on one stream)
        shared = ("k_cache", "v_cache", "seq_offsets", "prefill_r2s", "prompt_static", "tok", "pos",
                  "out_tokens", "sites_buf", "cur_step", "h_trace")
        if share is not None:
            for a in shared:
                setattr(self, a, getattr(share, a))
        else:
            self.k_cache = [torch.zeros((batch, H, self.Tmax, D), dtype=dtype, device=dv)
                            for _ in range(cfg.n_layers)]
            self.v_cache = [torch.zeros((batch, H, self.Tmax, D), dtype=dtype, device=dv)
                            for _ in range(cfg.n_layers)]
            self.seq_offsets = torch.arange(0, (batch + 1) * prompt_len, prompt_len, dtype=torch.int32, device=dv)
            # prefill row -> sequence (supplied-bounds check of the first token)
            self.prefill_r2s = torch.arange(batch * prompt_len, dtype=torch.int32, device=dv) // prompt_len
            # decode-step static buffers (CUDA-graph inputs/outputs)
            self.prompt_static = torch.zeros((batch, prompt_len), dtype=torch.int64, device=dv)
            self.tok = torch.zeros(batch, dtype=torch.int64, device=dv)
            self.pos = torch.zeros(1, dtype=torch.int64, device=dv)
            self.out_tokens = torch.zeros((batch, gen_len), dtype=torch.int64, device=dv)
            # stable site buffer: graphs captured with faults bake in its address, so
            # a campaign rewrites it per batch (set_sites / make_sites) and replays
            self.sites_buf = torch.zeros(batch * F2.SITE_BYTES, dtype=torch.uint8, device=dv)
            self.cur_step = torch.zeros(1, dtype=torch.int32, device=dv)
            # last-position hidden state (before the final norm) of every generated
            # token [G, B, hidden]: the campaign's deviation proxy reads it
            self.h_trace = torch.zeros((gen_len, batch, h), dtype=dtype, device=dv)
        self.graph_prefill = True   # first-token pass as a CUDA graph (False: eager)
        self.sites = None        # optional fault sites (uint8 [B*24]); site i = sequence i
        # caller-supplied ("offline") bounds [n_crit, B, 2] (set_supplied_bounds):
        # the first-token bound sweep is skipped and the prefill outputs are
        # checked against them like every later token
        self.supplied_bounds = None
        self._profile_keys = None
        self.graphs = {}
        self._pool = torch.cuda.graph_pool_handle() if self.device.type == "cuda" else None   # shared by all graphs
        self.time_phases = False
        self._phase_events = []
        self.mode = "fused"
        self._nv = None          # NaN-vulnerable profiling counts [n_layers * n_lin, B] (profile_nan_vulnerable)
        if cfg.arch == "llama":
            inv = 1.0 / (10000 ** (torch.arange(0, D, 2, device=dv, dtype=torch.float32) / D))
            t = torch.arange(self.Tmax, device=dv, dtype=torch.float32)
            fr = torch.outer(t, inv)
            self.rope_cos = torch.cat([fr.cos(), fr.cos()], -1).to(dtype)
            self.rope_sin = torch.cat([fr.sin(), fr.sin()], -1).to(dtype)

    # ------------------------------------------------------------ helpers
    def _norm(self, x, w, b):
        n = x.shape[-1]
        if self.host_norm and x.is_cuda and n % 8 == 0 and n <= 8192:
            x2 = x.reshape(-1, n)
            if x2.stride(-1) != 1:
                x2 = x2.contiguous()
            y = torch.empty((x2.shape[0], n), dtype=x.dtype, device=x.device)
            try:
                F2.host_norm(x2, w, y, bias=b if self.cfg.arch == "opt" else None,
                             eps=1e-5 if self.cfg.arch == "opt" else 1e-6, rms=self.cfg.arch != "opt")
                return y.view(*x.shape[:-1], n)
            except ValueError:   # tensors the host kernel does not take: torch's norm
                pass
        if self.cfg.arch == "opt":
            return F.layer_norm(x, (x.shape[-1],), w, b, 1e-5)
        return F.rms_norm(x, (x.shape[-1],), w, 1e-6)

    def _act(self, a, b=None):
        """relu(a) (OPT) or silu(a) * b (Llama) ahead of the critical fc2 /
        down_proj layer; libft2's host kernel triggers PDL dependents."""
        n = a.shape[-1]
        # decode-sized tensors only: there the launch latency is what PDL
        # hides; at prefill size (4096 x 8192) torch's unrolled kernel is
        # faster than this one (measured +0.42 ms per OPT-1.3B prefill)
        if self.host_act and a.is_cuda and n % 8 == 0 and a.dim() == 2 and a.shape[0] <= 256 and \
                a.stride(-1) == 1 and \
                (b is None or (b.dim() == 2 and b.stride(-1) == 1)):
            y = torch.empty((a.shape[0], n), dtype=a.dtype, device=a.device)
            try:
                return F2.host_act(a, y, b=b, act="relu" if b is None else "silu_mul")
            except ValueError:   # tensors the host kernel does not take: torch's op
                pass
        return torch.relu(a) if b is None else F.silu(a) * b

    def _rope(self, x, pos_idx):
        cos = self.rope_cos[pos_idx].unsqueeze(1)
        sin = self.rope_sin[pos_idx].unsqueeze(1)
        d = x.shape[-1] // 2
        rot = torch.cat([-x[..., d:], x[..., :d]], -1)
        return x * cos + rot * sin

    def _crit_id(self, blk, name):
        return blk * len(self.crit_names) + self.crit_names.index(name)

    def _lin_id(self, blk, name):
        """Linear-layer id for fault sites: block-major over all linear layers."""
        return blk * len(self.lin_names) + self.lin_names.index(name)

    def _linear(self, x2, blk: Block, name: str, phase: str, step_for_sites=None):
        """One linear layer of the block; FT2 work on critical ones.

        phase "prefill": bounds from the first-token output (+ NaN/Inf correction).
        phase "decode":  check-and-clip according to self.mode.
        With self.sites set (fault-injection campaign; eager or per-step graphs), the
        site of each trial row is applied to the layer's bf16 output before the
        check (order GEMM -> bias -> bf16 -> inject -> check, readings A19/A20).
        """
        w, b = blk.w[name], blk.b[name]
        crit = name in self.crit_names
        sites = self.sites
        step = 0 if phase == "prefill" else (step_for_sites if step_for_sites is not None else 0)
        lid = self._lin_id(blk.idx, name) if sites is not None else 0
        if phase == "prefill":
            # prefill GEMMs are compute-bound (M = B*T); they run on cuBLAS in
            # every mode and FT2's first-token work is the bounds sweep below
            y = F.linear(x2, w, b)
            if sites is not None:
                F2.inject_faults(y, sites, lid, 0, base_row=self.seq_offsets, n_sites=self.B)
            if self._nv is not None:
                li = self._lin_id(blk.idx, name)
                F2.bounds_from_prefill(y, None, self._nv_ws, seq_offsets=self.seq_offsets, num_seqs=self.B,
                                       finalize=False, keys_out=self._nv_keys, nan_vulnerable_count=self._nv[li])
            if crit and self._profile_keys is not None:   # offline profiling: raw keys, all rows one range
                cid = self._crit_id(blk.idx, name)
                F2.bounds_from_prefill(y, None, self.state.ws, num_seqs=1, finalize=False,
                                       keys_out=self._profile_tmp)
                torch.maximum(self._profile_keys[cid], self._profile_tmp[0], out=self._profile_keys[cid])
            elif crit and self.mode != "off":
                cid = self._crit_id(blk.idx, name)
                st = self.state
                if self.supplied_bounds is not None:   # offline bounds: the first token is checked too
                    F2.protect(y, st.bounds[cid], row_to_seq=self.prefill_r2s, num_seqs=self.B,
                               corrected_count=st.corrected[cid])
                else:
                    F2.bounds_from_prefill(y, st.bounds[cid], st.ws, seq_offsets=self.seq_offsets, num_seqs=self.B,
                                           scale=self.scale, correct_nonfinite=True,
                                           nonfinite_count=st.nonfinite[cid])
            return y
        # decode.  The fused tcgen05 GEMM serves decode batches of up to
        # FUSED_MAX_M tokens (swap-AB, cluster split-K); larger decode batches
        # (the 256-trial campaign) would land on the persistent prefill kernel,
        # which has no split-K and starves the grid at M = 256 (measured 1.4-2.5x
        # slower than cuBLAS, profiles/r1_m256_probe.txt), so there "fused" runs
        # cuBLAS + ft2_protect and "fused_plain" plain cuBLAS.
        fused_ok = x2.shape[0] <= FUSED_MAX_M and name not in self.standalone_layers
        if not crit or self.mode in ("off", "standalone") or not fused_ok:
            if crit and not fused_ok and self.mode == "fused":
                y = F.linear(x2, w, b)
                if sites is not None:
                    F2.inject_faults(y, sites, lid, step, n_sites=self.B)
                cid = self._crit_id(blk.idx, name)
                F2.protect(y, self.state.bounds[cid], num_seqs=self.B, corrected_count=self.state.corrected[cid])
                return y
            y = F.linear(x2, w, b)
            if sites is not None:
                F2.inject_faults(y, sites, lid, step, n_sites=self.B)
            if crit and self.mode == "standalone":
                cid = self._crit_id(blk.idx, name)
                st = self.state
                F2.protect(y, st.bounds[cid], num_seqs=self.B, corrected_count=st.corrected[cid])
            return y
        cid = self._crit_id(blk.idx, name)
        st = self.state
        y = torch.empty((x2.shape[0], w.shape[0]), dtype=self.dt, device=x2.device)
        mode = (FT2_GEMM_CHECK if self.mode == "fused" else FT2_GEMM_PLAIN) | FT2_GEMM_W_STATIC
        F2.protect_fused_gemm(x2, w, y, bias=b, mode=mode, bounds=st.bounds[cid], num_seqs=self.B,
                              corrected_count=st.corrected[cid], sites=sites, n_sites=self.B if sites is not None else None,
                              cur_layer=lid, cur_step=step, l2_prefetch=self._next_fused_w(blk, name))
        return y

    def _fused_gemm_order(self):
        """(block, layer-or-group name) of every decode GEMM that runs on the
        fused tcgen05 kernel, in execution order (the critical layers, or their
        fused q/k/v / gate/up groups)."""
        order = []
        for blk in self.blocks:
            for name in self.lin_names:
                if name not in self.crit_names:
                    continue
                g = next((g for g, ns in blk.groups.items() if name in ns and self._group_ok(blk, g)), None)
                order.append((blk, g if g is not None else name))
        return order

    def _next_fused_w(self, blk, name):
        """Weights of the fused GEMM that follows (blk, name) in a decode step
        (the first one of the next step after the last), as an L2 prefetch hint."""
        if not self.l2_prefetch:
            return None
        if getattr(self, "_next_w", None) is None:
            order = self._fused_gemm_order()
            w_of = lambda b_, n_: b_.wf[n_] if n_ in b_.wf else b_.w[n_]
            nxt = {(b_.idx, n_): order[(i + 1) % len(order)] for i, (b_, n_) in enumerate(order)}
            self._next_w = {k: w_of(*v) for k, v in nxt.items()
                            if not self.l2_prefetch_after_attn or v[1] in ("out_proj", "o_proj")}
        return self._next_w.get((blk.idx, name))

    def _group_ok(self, blk: Block, g: str) -> bool:
        """A fused group runs as one GEMM when fusion is on, no fault sites are
        armed, and at most one of its layers is protected (one column range)."""
        if not self.fuse_proj or g not in blk.groups:
            return False
        if self.sites is not None:
            raise ValueError("fault sites address single linear layers: build the runner with fuse_proj=False")
        return sum(n in self.crit_names for n in blk.groups[g]) <= 1

    def _linear_group(self, x2, blk: Block, g: str, phase: str, step_for_sites=None):
        """A horizontally fused projection group (qkv / gate_up): one GEMM whose
        output columns are the group's layers side by side.  FT2 work applies
        to the protected layer's column slice only: first-token bounds on the
        slice (strided view), and in decode the check in the fused GEMM's
        epilogue restricted to [col_begin, col_end) -- the other columns are
        written unchecked.  Returns the per-layer column views."""
        w, b = blk.wf[g], blk.bf[g]
        names = blk.groups[g]
        offs = [0]
        for n in names:
            offs.append(offs[-1] + blk.w[n].shape[0])
        crit = [i for i, n in enumerate(names) if n in self.crit_names]
        ci = crit[0] if crit else None
        st = self.state
        M = x2.shape[0]
        if phase == "prefill":
            y = F.linear(x2, w, b)
            if self._nv is not None:
                for i, n in enumerate(names):
                    F2.bounds_from_prefill(y[:, offs[i]:offs[i + 1]], None, self._nv_ws, seq_offsets=self.seq_offsets,
                                           num_seqs=self.B, finalize=False, keys_out=self._nv_keys,
                                           nan_vulnerable_count=self._nv[self._lin_id(blk.idx, n)])
            if ci is not None and self.mode != "off":
                cid = self._crit_id(blk.idx, names[ci])
                if self.supplied_bounds is not None or self._profile_keys is not None:
                    raise ValueError("supplied / profiled bounds need fuse_proj=False")
                F2.bounds_from_prefill(y[:, offs[ci]:offs[ci + 1]], st.bounds[cid], st.ws, seq_offsets=self.seq_offsets,
                                       num_seqs=self.B, scale=self.scale, correct_nonfinite=True,
                                       nonfinite_count=st.nonfinite[cid])
        elif ci is not None and self.mode in ("fused", "fused_plain") and M <= FUSED_MAX_M:
            cid = self._crit_id(blk.idx, names[ci])
            y = torch.empty((M, w.shape[0]), dtype=self.dt, device=x2.device)
            mode = (FT2_GEMM_CHECK if self.mode == "fused" else FT2_GEMM_PLAIN) | FT2_GEMM_W_STATIC
            F2.protect_fused_gemm(x2, w, y, bias=b, mode=mode, col_begin=offs[ci], col_end=offs[ci + 1],
                                  bounds=st.bounds[cid], num_seqs=self.B, corrected_count=st.corrected[cid],
                                  l2_prefetch=self._next_fused_w(blk, g))
        else:
            y = F.linear(x2, w, b)
            if ci is not None and (self.mode == "standalone" or (self.mode == "fused" and M > FUSED_MAX_M)):
                cid = self._crit_id(blk.idx, names[ci])
                F2.protect(y[:, offs[ci]:offs[ci + 1]], st.bounds[cid], num_seqs=self.B,
                           corrected_count=st.corrected[cid])
        return [y[:, offs[i]:offs[i + 1]] for i in range(len(names))]

    # ------------------------------------------------------------ forward
    def _block(self, blk: Block, x, phase, pos_idx=None, step=None):
        cfg = self.cfg
        B = self.B
        H, D = cfg.n_heads, cfg.head_dim
        T = x.shape[1]
        h = self._norm(x, blk.ln1_w, blk.ln1_b)
        h2 = h.reshape(-1, cfg.hidden)
        if self._group_ok(blk, "qkv"):
            q, k, v = self._linear_group(h2, blk, "qkv", phase, step)
        else:
            # v first: the protected projection then follows a torch kernel
            # (layer norm) instead of a cuBLAS GEMM, after which the tcgen05
            # GEMM's launch measured 1.3 us slower (tools/after_cublas_probe.py);
            # the three projections are independent, so the order is free
            v = self._linear(h2, blk, "v_proj", phase, step)
            q = self._linear(h2, blk, "q_proj", phase, step)
            k = self._linear(h2, blk, "k_proj", phase, step)
        q = q.view(B, T, H, D).transpose(1, 2)
        k = k.view(B, T, H, D).transpose(1, 2)
        v = v.view(B, T, H, D).transpose(1, 2)
        if cfg.arch == "llama":
            q = self._rope(q, pos_idx)
            k = self._rope(k, pos_idx)
        kc, vc = self.k_cache[blk.idx], self.v_cache[blk.idx]
        if phase == "prefill":
            kc[:, :, :T] = k
            vc[:, :, :T] = v
            a = F.scaled_dot_product_attention(q, k, v, is_causal=True)
        else:
            kc.index_copy_(2, self.pos, k)
            vc.index_copy_(2, self.pos, v)
            # one fused attention kernel over the whole (masked) cache
            a = F.scaled_dot_product_attention(q, kc, vc, attn_mask=self._mask)
        a = a.transpose(1, 2).reshape(-1, cfg.hidden)
        o_name = "out_proj" if cfg.arch == "opt" else "o_proj"
        x = x + self._linear(a, blk, o_name, phase, step).view(B, T, -1)
        h = self._norm(x, blk.ln2_w, blk.ln2_b).reshape(-1, cfg.hidden)
        if cfg.arch == "opt":
            f = self._act(self._linear(h, blk, "fc1", phase, step))
            y = self._linear(f, blk, "fc2", phase, step)
        else:
            if self._group_ok(blk, "gate_up"):
                g, u = self._linear_group(h, blk, "gate_up", phase, step)
            else:
                g = self._linear(h, blk, "gate_proj", phase, step)
                u = self._linear(h, blk, "up_proj", phase, step)
            y = self._linear(self._act(g, u), blk, "down_proj", phase, step)
        return x + y.view(B, T, -1)

    def _embed(self, ids, pos_idx):
        x = self.embed[ids]
        if self.cfg.arch == "opt":
            x = x + self.pos_embed[pos_idx + 2]
        return x

    def _logits_next(self, x_last):
        h = self._norm(x_last, self.lnf_w, self.lnf_b)
        return torch.argmax(F.linear(h, self.lm_head).float(), dim=-1)

    def prefill(self, prompt_ids):
        """First-token generation: FT2 bounds for every critical layer."""
        B, T = prompt_ids.shape
        pos = torch.arange(T, device=self.device)
        x = self._embed(prompt_ids, pos.unsqueeze(0).expand(B, T))
        pidx = pos.unsqueeze(0).expand(B, T)
        for blk in self.blocks:
            x = self._block(blk, x, "prefill", pos_idx=pidx, step=0)
        self.h_trace[0].copy_(x[:, -1])
        nxt = self._logits_next(x[:, -1])
        return nxt

    def _decode_step(self):
        """One decode step on static buffers (graph-capturable)."""
        pidx = self.pos.view(1, 1).expand(self.B, 1)
        ar = torch.arange(self.Tmax, device=self.device)
        self._mask = torch.where(ar <= self.pos, 0.0, float("-inf")).to(self.dt).view(1, 1, 1, -1)
        x = self._embed(self.tok.view(self.B, 1), pidx)
        for blk in self.blocks:
            x = self._block(blk, x, "decode", pos_idx=pidx, step=self._site_step)
        gi = (self.pos - self.T + 1).clamp_(0, self.G - 1)
        self.h_trace.index_copy_(0, gi, x[:, -1].unsqueeze(0))
        nxt = self._logits_next(x[:, -1])
        self.out_tokens.index_copy_(1, gi, nxt.view(self.B, 1))
        self.tok.copy_(nxt)
        self.pos.add_(1)

    def with_coverage(self, coverage: str) -> "Runner":
        """A runner protecting another layer set (Table 1) over the
        SAME weights, caches and site buffer (no copy): its own bounds,
        counters and CUDA graphs.  Used for paired coverage comparisons."""
        return Runner(self.cfg, self.B, self.T, self.G, device=self.device, scale=self.scale, coverage=coverage,
                      fuse_proj=self.fuse_proj, share=self, dtype=self.dt)

    def set_supplied_bounds(self, bounds):
        """Caller-supplied ("offline") bounds, bf16 [n_crit, B, 2] or [n_crit, 2]
        (broadcast over the batch), or None to return to first-token bounds.
        With bounds supplied the prefill skips FT2's first-token bound sweep
        and checks the protected prefill outputs against them instead (range
        restriction with fixed bounds, as the offline-profiled schemes
        PAPER.md L116 / L286 compare against)."""
        if bounds is None:
            self.supplied_bounds = None
            return
        b = bounds.to(device=self.device, dtype=self.dt)
        if b.dim() == 2:
            b = b.unsqueeze(1).expand(self.n_crit, self.B, 2)
        assert tuple(b.shape) == (self.n_crit, self.B, 2), b.shape
        self.supplied_bounds = b.contiguous().clone()

    def profile_offline_bounds(self, prompt_batches, scale=None):
        """Offline bound profiling (the baseline FT2 replaces, PAPER.md L116,
        L286): run unprotected first-token passes over `prompt_batches` (each
        [B, T] token ids) and keep, per protected layer, the min / max over
        every finite output of every batch, widened by `scale` (default the
        runner's, 2).  Exact: raw order keys max-combined across batches, then
        ft2_bounds_finalize.  Returns bf16 [n_crit, 2]."""
        st = self.state
        self._profile_keys = torch.full((self.n_crit, 2), -1, dtype=torch.int32, device=self.device)
        self._profile_tmp = torch.zeros((1, 2), dtype=torch.int32, device=self.device)
        mode, self.mode = self.mode, "off"
        try:
            for ids in prompt_batches:
                self.prefill(ids.to(self.device))
        finally:
            self.mode = mode
        out = torch.zeros((self.n_crit, 2), dtype=self.dt, device=self.device)
        F2.bounds_finalize(self._profile_keys, out, scale=self.scale if scale is None else scale)
        self._profile_keys = None
        return out

    def set_sites(self, sites):
        """Fault sites for the next generate() calls (uint8 [B*24], site i =
        sequence i), copied into the stable sites_buf; None = fault-free."""
        if sites is None:
            self.sites = None
            return
        if sites.data_ptr() != self.sites_buf.data_ptr():
            self.sites_buf.copy_(sites.view(torch.uint8).reshape(-1)[: self.sites_buf.numel()])
        self.sites = self.sites_buf

    def make_sites(self, seed, trial0, fault_model, step_policy=0):
        """ft2_make_fault_sites for trials [trial0, trial0 + B) straight into
        sites_buf (one site per batch row), and arm them."""
        F2.make_fault_sites(seed, trial0, self.B, fault_model, self.cfg.linear_widths(), n_steps=self.G - 1,
                            prompt_len=self.T, step_policy=step_policy, out=self.sites_buf, device=self.device)
        self.sites = self.sites_buf

    def _graph(self, mode, step_for_sites):
        """CUDA graph of one decode step.  Fault-free: one graph per mode.  With
        fault sites armed: one graph per (mode, decode step t), since the
        injection matches sites against the host-side step index."""
        faulty = self.sites is not None
        key = (mode, step_for_sites if faulty else None, faulty)
        if key not in self.graphs:
            self.mode = mode
            self._site_step = step_for_sites if faulty else None
            st = self.state
            s = torch.cuda.Stream()
            s.wait_stream(torch.cuda.current_stream())
            with torch.cuda.stream(s):
                save = (self.tok.clone(), self.pos.clone(), self.out_tokens.clone(), st.corrected.clone(),
                        st.nonfinite.clone())
                for _ in range(2):   # warm-up (allocations, cuBLAS handles)
                    self._decode_step()
                self._restore(save)
            torch.cuda.current_stream().wait_stream(s)
            g = torch.cuda.CUDAGraph()
            n0 = F2.launch_count()
            with torch.cuda.graph(g, pool=self._pool):
                self._decode_step()
            self.graphs[key] = (g, F2.launch_count() - n0)
            self._restore(save)
        return self.graphs[key]

    def _restore(self, save):
        self.tok.copy_(save[0]); self.pos.copy_(save[1]); self.out_tokens.copy_(save[2])
        self.state.corrected.copy_(save[3]); self.state.nonfinite.copy_(save[4])

    def _prefill_graph(self, mode):
        """CUDA graph of the whole first-token pass (embedding, 24 blocks with
        the FT2 bound sweeps on the critical layers, LM head, first token) on
        the static prompt buffer; one per mode."""
        key = ("prefill", mode, self.sites is not None, self.supplied_bounds is not None)
        if key not in self.graphs:
            self.mode = mode
            self._site_step = None

            def body():
                first = self.prefill(self.prompt_static)
                self.out_tokens[:, 0] = first
                self.tok.copy_(first)
                self.pos.fill_(self.T)

            s = torch.cuda.Stream()
            s.wait_stream(torch.cuda.current_stream())
            with torch.cuda.stream(s):
                body()   # warm-up (allocations, cuBLAS/cuDNN plans)
            torch.cuda.current_stream().wait_stream(s)
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, pool=self._pool):
                body()
            self.graphs[key] = g
        return self.graphs[key]

    def ft2_launches_per_request(self, mode):
        """Library kernels launched by one generate() in `mode` (prefill + decode replays)."""
        if mode == "off":
            return 0
        per_prefill = self.n_crit
        g, per_step = self._graph(mode, None)
        return per_prefill + per_step * (self.G - 1)

    def generate(self, prompt_ids, mode="fused", use_graph=True):
        """Greedy generation of G tokens (1 first token + G-1 decode steps).
        With fault sites armed (set_sites / make_sites) and use_graph, every
        decode step t replays its own captured graph (captured on first use)."""
        self.mode = mode
        self._site_step = None
        faulty = self.sites is not None
        if use_graph and self.graph_prefill:
            pg = self._prefill_graph(mode)   # capture (and its warm-up) before the counters reset
        self.state.reset_counters()
        if self.supplied_bounds is not None:
            self.state.bounds.copy_(self.supplied_bounds)
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(3)] if self.time_phases else None
        if ev:
            ev[0].record()
        if use_graph and self.graph_prefill:
            self.prompt_static.copy_(prompt_ids, non_blocking=True)
            pg.replay()
        else:
            first = self.prefill(prompt_ids)
            self.out_tokens[:, 0] = first
            self.tok.copy_(first)
            self.pos.fill_(self.T)
        if ev:
            ev[1].record()
        if use_graph and faulty:
            for t in range(1, self.G):
                g, _ = self._graph(mode, t)   # decode step t (0 = prefill / first token)
                g.replay()
            self.mode = mode
        elif use_graph:
            g, _ = self._graph(mode, None)
            self.mode = mode
            for _ in range(self.G - 1):
                g.replay()
        else:
            for t in range(1, self.G):
                self._site_step = t   # decode step t (0 = prefill / first token)
                self._decode_step()
            self._site_step = None
        if ev:
            ev[2].record()
            self._phase_events.append(ev)
        return self.out_tokens

    def profile_nan_vulnerable(self, prompt_ids):
        """Share of NaN-vulnerable values in every linear layer's output.

        PAPER.md L202 / Fig. 8(b): a fault-free profiling run records, per
        linear layer, the percentage of output values in (-2,-1) U (1,2) --
        those a flip of the highest exponent bit turns into NaN (L185, Fig. 7);
        L212 names it the first proxy for layer criticality.  Runs one
        unprotected prefill (mode "off") and counts inside the bounds sweep.
        Returns (per-name share averaged over blocks and sequences, raw counts
        [n_layers, n_lin, B] as int64, elements per (layer, sequence) [n_lin]).
        """
        B = self.B
        n_lin = len(self.lin_names)
        self._nv = torch.zeros((self.cfg.n_layers * n_lin, B), dtype=torch.int32, device=self.device)
        self._nv_keys = torch.zeros((B, 2), dtype=torch.int32, device=self.device)
        self._nv_ws = F2.make_workspace(B, device=self.device)
        mode, self.mode = self.mode, "off"
        try:
            self.prefill(prompt_ids)
            torch.cuda.synchronize()
            counts = self._nv.view(self.cfg.n_layers, n_lin, B).to(torch.int64).cpu()
        finally:
            self._nv = None
            self.mode = mode
        elems = torch.tensor([o * self.T for _, o, _, _ in self.cfg.linears()], dtype=torch.int64)
        share = counts.sum(dim=(0, 2)).double() / (elems.double() * self.cfg.n_layers * B)
        return {n: float(share[i]) for i, n in enumerate(self.lin_names)}, counts, elems

    def phase_times(self):
        """(prefill ms, decode ms per step) averaged over the generate() calls
        since the last call (requires time_phases = True)."""
        torch.cuda.synchronize()
        if not self._phase_events:
            return None
        pre = sum(e[0].elapsed_time(e[1]) for e in self._phase_events) / len(self._phase_events)
        dec = sum(e[1].elapsed_time(e[2]) for e in self._phase_events) / len(self._phase_events) / max(1, self.G - 1)
        self._phase_events = []
        return pre, dec
