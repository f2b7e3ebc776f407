"""Critical-layer selection (R1) and protection-coverage tables -- ORACLE.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

PAPER.md L149 (Sec. 4, step 1), L212-L214 (Sec. 4.1.2, TA#5): "a layer is
deemed critical if no scaling operation or activation layer is present before
the next linear layer".  This module writes that heuristic out as a walk over
an explicit per-block operator graph and is pinned (tests/test_oracle_critical.py)
against Table 1.

Operator graphs, Fig. 1.  The operator order inside
each block is an external fact taken from the HF transformers sources in this
image: OPT ``q_proj(..)*scaling`` (modeling_opt.py:151) and
fc1 -> activation -> fc2 (:241-244); Llama ``down_proj(act_fn(gate_proj(x)) *
up_proj(x))`` (modeling_llama.py:183) and QK^T * scaling (:212); GPT-J fc_in
-> act -> fc_out with a parallel residual (modeling_gptj.py:375-377, 411).

Reading (R1): shielding ops are {activation, scaling (incl. the
attention-score scaling / softmax)}.  Not counted: residual add,
LayerNorm/RMSNorm, RoPE, reshape, dropout, P*V, the elementwise gate product,
bias.  A linear layer is critical iff every dataflow path from its output to
the next linear layer(s) is free of shielding ops.
"""
from __future__ import annotations

SHIELDING = frozenset({"activation", "scale", "softmax"})

# Each graph: node -> (kind, [successor nodes]).  "linear" nodes are the
# candidates; "next_*" linear nodes stand for the following block's layers.


def _opt_graph():
    """OPT-style block (Fig. 1(a)); q is scaled at q_proj (modeling_opt.py:151)."""
    return {
        "ln1": ("norm", ["q_proj", "k_proj", "v_proj"]),
        "q_proj": ("linear", ["q_scale"]),
        "q_scale": ("scale", ["qk"]),
        "k_proj": ("linear", ["qk"]),
        "qk": ("matmul", ["softmax"]),
        "softmax": ("softmax", ["pv"]),
        "v_proj": ("linear", ["pv"]),
        "pv": ("matmul", ["out_proj"]),
        "out_proj": ("linear", ["res1"]),
        "res1": ("residual", ["ln2", "res2"]),
        "ln2": ("norm", ["fc1"]),
        "fc1": ("linear", ["act"]),
        "act": ("activation", ["fc2"]),
        "fc2": ("linear", ["res2"]),
        "res2": ("residual", ["next_ln1"]),
        "next_ln1": ("norm", ["next_q", "next_k", "next_v"]),
        "next_q": ("linear", []), "next_k": ("linear", []), "next_v": ("linear", []),
    }


def _gptj_graph():
    """GPT-J block: parallel residual, attention and MLP both read ln(x)
    (modeling_gptj.py:375-377, 411); QK^T scaled before softmax."""
    return {
        "ln1": ("norm", ["q_proj", "k_proj", "v_proj", "fc_in"]),
        "q_proj": ("linear", ["rope_q"]),
        "rope_q": ("rope", ["qk"]),
        "k_proj": ("linear", ["rope_k"]),
        "rope_k": ("rope", ["qk"]),
        "qk": ("matmul", ["qk_scale"]),
        "qk_scale": ("scale", ["softmax"]),
        "softmax": ("softmax", ["pv"]),
        "v_proj": ("linear", ["pv"]),
        "pv": ("matmul", ["out_proj"]),
        "out_proj": ("linear", ["res"]),
        "fc_in": ("linear", ["act"]),
        "act": ("activation", ["fc_out"]),
        "fc_out": ("linear", ["res"]),
        "res": ("residual", ["next_ln1"]),
        "next_ln1": ("norm", ["next_q", "next_k", "next_v", "next_fc_in"]),
        "next_q": ("linear", []), "next_k": ("linear", []), "next_v": ("linear", []),
        "next_fc_in": ("linear", []),
    }


def _llama_graph():
    """Llama/Qwen2 block (Fig. 1(b)); QK^T * scaling (modeling_llama.py:212);
    down(act(gate(x)) * up(x)) (modeling_llama.py:183)."""
    return {
        "ln1": ("norm", ["q_proj", "k_proj", "v_proj"]),
        "q_proj": ("linear", ["rope_q"]),
        "rope_q": ("rope", ["qk"]),
        "k_proj": ("linear", ["rope_k"]),
        "rope_k": ("rope", ["qk"]),
        "qk": ("matmul", ["qk_scale"]),
        "qk_scale": ("scale", ["softmax"]),
        "softmax": ("softmax", ["pv"]),
        "v_proj": ("linear", ["pv"]),
        "pv": ("matmul", ["o_proj"]),
        "o_proj": ("linear", ["res1"]),
        "res1": ("residual", ["ln2", "res2"]),
        "ln2": ("norm", ["gate_proj", "up_proj"]),
        "gate_proj": ("linear", ["act"]),
        "act": ("activation", ["gate_mul"]),
        "up_proj": ("linear", ["gate_mul"]),
        "gate_mul": ("elementwise_mul", ["down_proj"]),
        "down_proj": ("linear", ["res2"]),
        "res2": ("residual", ["next_ln1"]),
        "next_ln1": ("norm", ["next_q", "next_k", "next_v"]),
        "next_q": ("linear", []), "next_k": ("linear", []), "next_v": ("linear", []),
    }


GRAPHS = {"opt": _opt_graph, "gptj": _gptj_graph, "llama": _llama_graph, "qwen2": _llama_graph}

# Canonical layer names of Table 1 per architecture node name.
TABLE1_NAME = {
    "q_proj": "Q_PROJ", "k_proj": "K_PROJ", "v_proj": "V_PROJ", "out_proj": "OUT_PROJ",
    "o_proj": "OUT_PROJ", "fc1": "FC1", "fc_in": "FC1", "fc2": "FC2", "fc_out": "FC2",
    "up_proj": "UP_PROJ", "gate_proj": "GATE_PROJ", "down_proj": "DOWN_PROJ",
}


def _paths_clean(graph, start):
    """True iff every path from ``start``'s output to the next linear node
    passes no shielding op."""
    def walk(node, seen):
        kind, succ = graph[node]
        if node != start and kind == "linear":
            return True  # reached the next linear layer on a clean path
        if node != start and kind in SHIELDING:
            return False
        if not succ:
            return True
        ok = True
        for s in succ:
            if s in seen:
                continue
            ok = ok and walk(s, seen | {s})
        return ok
    return walk(start, {start})


def critical_layers(arch: str):
    """Dict layer-name -> critical (bool) for the block of ``arch``."""
    g = GRAPHS[arch]()
    out = {}
    for node, (kind, _) in g.items():
        if kind == "linear" and not node.startswith("next_"):
            out[node] = _paths_clean(g, node)
    return out


# Block linear-layer order used for layer ids (fault sites, protected lists).
BLOCK_LINEARS = {
    "opt": ["q_proj", "k_proj", "v_proj", "out_proj", "fc1", "fc2"],
    "gptj": ["q_proj", "k_proj", "v_proj", "out_proj", "fc_in", "fc_out"],
    "llama": ["q_proj", "k_proj", "v_proj", "o_proj", "gate_proj", "up_proj", "down_proj"],
    "qwen2": ["q_proj", "k_proj", "v_proj", "o_proj", "gate_proj", "up_proj", "down_proj"],
}

# Table 1 protection coverage of the comparison methods,
# transcribed as data (NEXT(4) coverage masks; their results are out of scope).
TABLE1_COVERAGE = {
    "Ranger": set(),  # activation layers only, no linear layer (L164, L315)
    "MaxiMals": {"OUT_PROJ", "FC2", "DOWN_PROJ"},
    "GlobalClipper": {"V_PROJ", "OUT_PROJ"},
    "FT2": {"V_PROJ", "OUT_PROJ", "FC2", "UP_PROJ", "DOWN_PROJ"},
}

# Table 1 "Critical Layer" column.
TABLE1_CRITICAL = {
    "K_PROJ": False, "Q_PROJ": False, "V_PROJ": True, "OUT_PROJ": True, "FC1": False,
    "FC2": True, "UP_PROJ": True, "GATE_PROJ": False, "DOWN_PROJ": True,
}
